// Peer-memory verdict / result exchange between ranks.
//
// Every rank owns one "exchange region" (cudaMalloc, exported with cudaIpcGetMemHandle and
// mapped by every peer with cudaIpcOpenMemHandle; over NVLink 5 / NVSwitch on an 8xB200 box).
// Regions have the same layout on every rank:
//
//   sig  [2 parity][3 kind][64 src] u64      kind 0: verdict planes of epoch e are in place
//                                            kind 1: result slots of epoch e are final
//                                            kind 2: slice sums of epoch e are final
//   board[2 parity][world src][nwords] uint4  per 32 txns: conflict-bit planes {UA,WAW,RAW,WAR}
//   res  [2 parity][nres] i64                the rank's own result slots (peers pull them)
//   rsum [2 parity][nres] i64                slice q of the summed slots (rank q computes it)
//   b8   [2 parity][world src][max_txns] u8  sharded batches: conflict bits of global rank g
//   rb   [2 parity][max_txns] {i64, i64}     sharded batches: (c_id, C_BALANCE) of a remote-
//                                            customer Payment of global rank g, for its home rank
//
// Rank q's batch e: detect -> k_xput stores its planes into board[e&1][q] of EVERY region
// (its own included) and, after a system-scope fence, sig[e&1][0][q] = e<<3 | err bits.
// k_xcombine waits until all world signals of epoch e are in ITS region, ORs the planes and
// writes the final status (identical on all ranks).  After write-back, k_xsig_res publishes
// sig[e&1][1][q] = e; the result sum is a reduce-scatter + all-gather over peer memory:
// k_xrs waits for every rank's kind-1 signal, sums slice q of the slots over all ranks into
// rsum and raises kind 2; k_xag waits for every kind-2 signal and gathers the other slices.
// Each rank pulls 2 (world-1)/world of the slot array -- what a ring allreduce moves.
//
// Sharded TPC-C batches (include/ltpg.h) exchange only what crosses ranks: k_xput_sharded stores
// the bits of every shard txn that touches several ranks into b8[e&1][q][g] of each other rank
// it touches, and a remote-customer Payment's (c_id, C_BALANCE) -- computed by the customer's
// rank -- into rb[e&1][g] of its home rank; then the kind-0 signal as above.  k_xcombine_sharded
// ORs the bytes of the ranks each txn touches and fills the home rank's result slots; there is
// no result sum (every result slot is final on its home rank).
//
// Buffer reuse is safe with two parities: rank q can only write parity (e&1) again in batch
// e+2, which it reaches after its combine of batch e+1, which waited for every peer's
// verdict signal of e+1 -- sent by each peer after it finished its combine / sum of batch e
// (a peer reads my res in its k_xrs and my rsum in its k_xag of batch e, both before its
// detection of batch e+1).
#pragma once
#include <cstdint>

#include <cuda_runtime.h>

namespace ltpg {

constexpr uint32_t NSIG = 3;  // signal kinds per parity

struct XLayout {
  uint64_t nwords = 0, nres = 0;
  uint32_t world = 1;
  uint64_t off_board = 0, off_res = 0, off_rsum = 0, off_b8 = 0, off_rb = 0, bytes = 0;
  uint32_t max_txns = 0;
  void init(uint32_t max_txns_, uint64_t nres_, uint32_t world_) {
    world = world_;
    max_txns = max_txns_;
    nwords = (max_txns + 31) / 32;
    nres = nres_;
    off_board = 2 * NSIG * 64 * sizeof(uint64_t);
    off_res = off_board + 2ull * world * nwords * 16;
    off_res = (off_res + 255) & ~255ull;
    off_rsum = off_res + 2ull * nres * sizeof(long long);
    off_b8 = off_rsum + 2ull * nres * sizeof(long long);
    off_rb = (off_b8 + 2ull * world * max_txns + 255) & ~255ull;
    bytes = off_rb + 2ull * max_txns * 16;
  }
};

struct XPeers {
  char* base[64];  // region of each rank, mapped into this process (own region included)
};

// after detect: local per-txn conflict bits -> planes in every region, then the signal
void launch_xput(const uint8_t* lflag, const uint32_t* err, uint32_t n, const XPeers& peers, const XLayout& L,
                 uint32_t rank, uint32_t epoch, uint32_t* done_counter, cudaStream_t s);
// wait for every rank's verdict of `epoch`, OR the planes -> status; OR of the error bits
// -> *err (this rank's partition word) and *err_all
void launch_xcombine(char* own, const XLayout& L, uint32_t n, uint32_t epoch, bool reorder, uint8_t* status,
                     uint32_t* err, uint32_t* err_all, cudaStream_t s);
// sharded TPC-C batch, after detect: bits of the txns touching other ranks + remote-customer
// Payment results -> the peers' regions, then the signal.  pmask / grank / lflag: per shard txn
void launch_xput_sharded(const uint8_t* lflag, const uint32_t* pmask, const uint32_t* grank, const uint8_t* ptype,
                         const uint8_t* params, const long long* res, const uint32_t* err, uint32_t n,
                         const XPeers& peers, const XLayout& L, uint32_t rank, uint32_t nw, uint32_t epoch,
                         uint32_t* done_counter, cudaStream_t s);
// wait for every rank's signal of `epoch`; status[i] from the OR of the bits of the ranks txn i
// touches; the home rank of a remote-customer Payment takes its result slots 0/1 from rb
void launch_xcombine_sharded(char* own, const XLayout& L, uint32_t n, uint32_t epoch, bool reorder, uint8_t* status,
                             const uint8_t* lflag, const uint32_t* pmask, const uint32_t* grank, const uint8_t* ptype,
                             const uint8_t* params, long long* res, uint32_t rank, uint32_t nw, uint32_t* err,
                             uint32_t* err_all, cudaStream_t s);
// after write-back: publish "my result slots of `epoch` are final"
void launch_xsig_res(const XPeers& peers, uint32_t rank, uint32_t world, uint32_t epoch, cudaStream_t s);
// reduce-scatter + all-gather of the result slots: out[i] = sum over ranks of their slot i
void launch_xsum(const XPeers& peers, const XLayout& L, uint64_t n_reads, uint32_t epoch, long long* out,
                 uint32_t* err, uint32_t rank, uint32_t* done_counter, cudaStream_t s);

}  // namespace ltpg
