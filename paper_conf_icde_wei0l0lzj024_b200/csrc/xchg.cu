// Peer-memory exchange kernels (protocol and layout: xchg.cuh), fused with the conflict test
// instead of a collective library's allreduce: global batches send a rank's verdicts as 4 bit
// planes per 32 txns (16 B) stored straight into every peer's region, i.e. (world-1) * n/2
// bytes per rank instead of a 4n-byte ring allreduce; sharded batches send one byte per
// cross-rank txn and peer.  The waiting side needs no host involvement.
#include <algorithm>

#include "ltpg_internal.cuh"
#include "xchg.cuh"

namespace ltpg {

namespace {

constexpr uint64_t SPIN_TIMEOUT_NS = 20ull * 1000 * 1000 * 1000;  // a peer that never arrives: fail

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t* sig_ptr(char* region, uint32_t par, uint32_t kind, uint32_t src) {
  return reinterpret_cast<uint64_t*>(region) + (par * NSIG + kind) * 64 + src;
}
__device__ __forceinline__ uint4* board_ptr(char* region, const XLayout& L, uint32_t par, uint32_t src) {
  return reinterpret_cast<uint4*>(region + L.off_board) + ((uint64_t)par * L.world + src) * L.nwords;
}

// Block-wide wait until sig[par][kind][src] of every src has reached `want` (value >> shift).
// Thread 0 spins with acquire loads; the barrier then orders the block's later loads.
// A block that times out sets ERR_EINTERNAL in *gave_up; the others then stop waiting too.
__device__ bool wait_all(char* own, uint32_t par, uint32_t kind, uint32_t world, uint64_t want, uint32_t shift,
                         uint32_t* errbits, uint32_t* gave_up) {
  __shared__ int ok;
  if (threadIdx.x == 0) {
    ok = 1;
    uint32_t e = 0;
    const uint64_t t0 = globaltimer();
    for (uint32_t src = 0; src < world; ++src) {
      uint64_t v;
      while (((v = ld_acquire_sys(sig_ptr(own, par, kind, src))) >> shift) < want) {
        if (globaltimer() - t0 > SPIN_TIMEOUT_NS || (*(volatile uint32_t*)gave_up & ERR_EINTERNAL)) {
          ok = 0;
          atomicOr(gave_up, ERR_EINTERNAL);
          break;
        }
        __nanosleep(200);
      }
      if (!ok) break;
      e |= (uint32_t)v & 7u;
    }
    if (errbits) *errbits = e;
  }
  __syncthreads();
  return ok != 0;
}

// One warp per 32 txns: ballots of the four conflict bits form the planes; lane 0 stores the
// 16-byte word into board[par][rank] of every region.  The last block to finish (counter)
// fences at system scope and raises the signal in every region.
__global__ void __launch_bounds__(256) k_xput(const uint8_t* __restrict__ lflag, const uint32_t* err, uint32_t n,
                                              XPeers peers, XLayout L, uint32_t rank, uint32_t epoch,
                                              uint32_t* done) {
  const uint32_t par = epoch & 1u;
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t f = r < n ? lflag[r] : 0u;
  const uint32_t ua = __ballot_sync(0xffffffffu, f & CF_UA), waw = __ballot_sync(0xffffffffu, f & CF_WAW);
  const uint32_t raw = __ballot_sync(0xffffffffu, f & CF_RAW), war = __ballot_sync(0xffffffffu, f & CF_WAR);
  const uint32_t w = r >> 5;
  if ((threadIdx.x & 31) < L.world && w < L.nwords) {  // lane q stores into region q
    const uint32_t q = threadIdx.x & 31;
    board_ptr(peers.base[q], L, par, rank)[w] = make_uint4(ua, waw, raw, war);
  }
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t prev = atomicAdd(done, 1u);
    if (prev == gridDim.x - 1) {  // every block's stores are fenced: publish
      __threadfence_system();
      const uint64_t v = ((uint64_t)epoch << 3) | (*err & 7u);
      for (uint32_t q = 0; q < L.world; ++q) st_release_sys(sig_ptr(peers.base[q], par, 0, rank), v);
      *done = 0;
    }
  }
}

__global__ void __launch_bounds__(256) k_xcombine(char* own, XLayout L, uint32_t n, uint32_t epoch, bool reorder,
                                                  uint8_t* status, uint32_t* err, uint32_t* err_all) {
  const uint32_t par = epoch & 1u;
  uint32_t e = 0;
  const bool ok = wait_all(own, par, 0, L.world, epoch, 3, &e, err_all);
  if (!ok) {
    if (threadIdx.x == 0) {
      atomicOr(err, ERR_EINTERNAL);
      atomicOr(err_all, ERR_EINTERNAL);
    }
    return;
  }
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    *err = e;
    *err_all = e;
  }
  if (r >= n) return;
  uint4 acc = make_uint4(0, 0, 0, 0);
  for (uint32_t src = 0; src < L.world; ++src) {
    const uint4 v = __ldcg(board_ptr(own, L, par, src) + (r >> 5));
    acc.x |= v.x, acc.y |= v.y, acc.z |= v.z, acc.w |= v.w;
  }
  const uint32_t b = r & 31;
  const uint32_t f = (((acc.x >> b) & 1u) ? CF_UA : 0u) | (((acc.y >> b) & 1u) ? CF_WAW : 0u) |
                     (((acc.z >> b) & 1u) ? CF_RAW : 0u) | (((acc.w >> b) & 1u) ? CF_WAR : 0u);
  status[r] = status_of_bits(f, reorder);
}

// ---- sharded TPC-C batches -------------------------------------------------------------------
__device__ __forceinline__ uint8_t* b8_ptr(char* region, const XLayout& L, uint32_t par, uint32_t src) {
  return reinterpret_cast<uint8_t*>(region + L.off_b8) + ((uint64_t)par * L.world + src) * L.max_txns;
}
__device__ __forceinline__ longlong2* rb_ptr(char* region, const XLayout& L, uint32_t par) {
  return reinterpret_cast<longlong2*>(region + L.off_rb) + (uint64_t)par * L.max_txns;
}
__device__ __forceinline__ uint32_t u16_at(const uint8_t* p, int off) {
  return p[off] | (uint32_t)p[off + 1] << 8;
}
// a Payment whose customer lives on another rank: (home rank, customer rank)
__device__ __forceinline__ bool remote_customer(const uint8_t* ptype, const uint8_t* params, uint32_t i, uint32_t nw,
                                                uint32_t world, uint32_t& home, uint32_t& cust) {
  if (ptype[i] != LTPG_PAYMENT) return false;
  const uint8_t* p = params + 128ull * i;
  home = part_of_w(u16_at(p, 0), nw, world);
  cust = part_of_w(u16_at(p, 4), nw, world);
  return home != cust;
}

__global__ void __launch_bounds__(256) k_xput_sharded(const uint8_t* __restrict__ lflag, const uint32_t* __restrict__ pmask,
                                                      const uint32_t* __restrict__ grank, const uint8_t* ptype,
                                                      const uint8_t* params, const long long* res, const uint32_t* err,
                                                      uint32_t n, XPeers peers, XLayout L, uint32_t rank, uint32_t nw,
                                                      uint32_t epoch, uint32_t* done) {
  const uint32_t par = epoch & 1u;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint32_t others = pmask[i] & ~(1u << rank);
    if (!others) continue;  // a txn of this rank only: its verdict is local
    const uint32_t g = grank[i];
    const uint8_t f = lflag[i];
    for (uint32_t m = others; m; m &= m - 1) b8_ptr(peers.base[__ffs(m) - 1], L, par, rank)[g] = f;
    uint32_t home, cust;
    if (remote_customer(ptype, params, i, nw, L.world, home, cust) && cust == rank)
      rb_ptr(peers.base[home], L, par)[g] = make_longlong2(res[4ull * i], res[4ull * i + 1]);
  }
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t prev = atomicAdd(done, 1u);
    if (prev == gridDim.x - 1) {  // every block's stores are fenced: publish
      __threadfence_system();
      const uint64_t v = ((uint64_t)epoch << 3) | (*err & 7u);
      for (uint32_t q = 0; q < L.world; ++q) st_release_sys(sig_ptr(peers.base[q], par, 0, rank), v);
      *done = 0;
    }
  }
}

__global__ void __launch_bounds__(256) k_xcombine_sharded(char* own, XLayout L, uint32_t n, uint32_t epoch,
                                                          bool reorder, uint8_t* status, const uint8_t* lflag,
                                                          const uint32_t* pmask, const uint32_t* grank,
                                                          const uint8_t* ptype, const uint8_t* params, long long* res,
                                                          uint32_t rank, uint32_t nw, uint32_t* err, uint32_t* err_all) {
  const uint32_t par = epoch & 1u;
  uint32_t e = 0;
  const bool ok = wait_all(own, par, 0, L.world, epoch, 3, &e, err_all);
  if (!ok) {
    if (threadIdx.x == 0) {
      atomicOr(err, ERR_EINTERNAL);
      atomicOr(err_all, ERR_EINTERNAL);
    }
    return;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    *err = e;
    *err_all = e;
  }
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    uint32_t f = lflag[i];
    const uint32_t others = pmask[i] & ~(1u << rank);
    if (others) {
      const uint32_t g = grank[i];
      for (uint32_t m = others; m; m &= m - 1) f |= __ldcg(b8_ptr(own, L, par, __ffs(m) - 1) + g);
      uint32_t home, cust;
      if (remote_customer(ptype, params, i, nw, L.world, home, cust) && home == rank) {
        const longlong2 v = __ldcg(rb_ptr(own, L, par) + g);
        res[4ull * i] = v.x;
        res[4ull * i + 1] = v.y;
        res[4ull * i + 2] = 0;
        res[4ull * i + 3] = 0;
      }
    }
    status[i] = status_of_bits(f, reorder);
  }
}

__global__ void k_xsig_res(XPeers peers, uint32_t rank, uint32_t world, uint32_t epoch) {
  __threadfence_system();
  const uint32_t par = epoch & 1u;
  if (threadIdx.x < world) st_release_sys(sig_ptr(peers.base[threadIdx.x], par, 1, rank), (uint64_t)epoch << 3);
}

// slice q of the slot array (rank q sums it): [q*S, min((q+1)*S, n)), S = ceil(n / world)
__device__ __forceinline__ void slice_of(uint64_t n, uint32_t world, uint32_t q, uint64_t& lo, uint64_t& hi) {
  const uint64_t S = (n + world - 1) / world;
  lo = min(n, (uint64_t)q * S);
  hi = min(n, lo + S);
}

// reduce-scatter: rsum[i] = sum over ranks of res[i] for i in this rank's slice; the last block
// to finish raises kind 2 in every region
__global__ void __launch_bounds__(256) k_xrs(XPeers peers, XLayout L, uint64_t n, uint32_t epoch, uint32_t* err,
                                             uint32_t rank, uint32_t* done) {
  const uint32_t par = epoch & 1u;
  const bool ok = wait_all(peers.base[rank], par, 1, L.world, epoch, 3, nullptr, err);
  if (ok) {
    const uint64_t off = L.off_res + (uint64_t)par * L.nres * sizeof(long long);
    long long* rsum = reinterpret_cast<long long*>(peers.base[rank] + L.off_rsum) + (uint64_t)par * L.nres;
    uint64_t lo, hi;
    slice_of(n, L.world, rank, lo, hi);
    for (uint64_t i = lo + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < hi; i += (uint64_t)gridDim.x * blockDim.x) {
      unsigned long long s = 0;
      for (uint32_t q = 0; q < L.world; ++q)
        s += (unsigned long long)__ldcg(reinterpret_cast<const long long*>(peers.base[q] + off) + i);
      rsum[i] = (long long)s;
    }
  } else if (threadIdx.x == 0) {
    atomicOr(err, ERR_EINTERNAL);
  }
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0 && atomicAdd(done, 1u) == gridDim.x - 1) {  // every block's sums are fenced
    __threadfence_system();
    for (uint32_t q = 0; q < L.world; ++q) st_release_sys(sig_ptr(peers.base[q], par, 2, rank), (uint64_t)epoch << 3);
    *done = 0;
  }
}

// all-gather: out[i] = rsum of slice owner(i), pulled from the owner's region
__global__ void __launch_bounds__(256) k_xag(XPeers peers, XLayout L, uint64_t n, uint32_t epoch, long long* out,
                                             uint32_t* err, uint32_t rank) {
  const uint32_t par = epoch & 1u;
  if (!wait_all(peers.base[rank], par, 2, L.world, epoch, 3, nullptr, err)) {
    if (threadIdx.x == 0) atomicOr(err, ERR_EINTERNAL);
    return;
  }
  const uint64_t S = (n + L.world - 1) / L.world;
  const uint64_t off = L.off_rsum + (uint64_t)par * L.nres * sizeof(long long);
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = __ldcg(reinterpret_cast<const long long*>(peers.base[i / S] + off) + i);
}

}  // namespace

void launch_xput(const uint8_t* lflag, const uint32_t* err, uint32_t n, const XPeers& peers, const XLayout& L,
                 uint32_t rank, uint32_t epoch, uint32_t* done, cudaStream_t s) {
  const uint32_t blocks = (n + 255) / 256 ? (n + 255) / 256 : 1;
  k_xput<<<blocks, 256, 0, s>>>(lflag, err, n, peers, L, rank, epoch, done);
  note_launch();
}

void launch_xcombine(char* own, const XLayout& L, uint32_t n, uint32_t epoch, bool reorder, uint8_t* status,
                     uint32_t* err, uint32_t* err_all, cudaStream_t s) {
  const uint32_t blocks = (n + 255) / 256 ? (n + 255) / 256 : 1;
  k_xcombine<<<blocks, 256, 0, s>>>(own, L, n, epoch, reorder, status, err, err_all);
  note_launch();
}

void launch_xput_sharded(const uint8_t* lflag, const uint32_t* pmask, const uint32_t* grank, const uint8_t* ptype,
                         const uint8_t* params, const long long* res, const uint32_t* err, uint32_t n,
                         const XPeers& peers, const XLayout& L, uint32_t rank, uint32_t nw, uint32_t epoch,
                         uint32_t* done, cudaStream_t s) {
  // grid-stride over the shard; the last block to finish raises the signals
  const uint32_t blocks = std::max<uint32_t>(1, std::min<uint32_t>((n + 255) / 256, 148 * 4));
  k_xput_sharded<<<blocks, 256, 0, s>>>(lflag, pmask, grank, ptype, params, res, err, n, peers, L, rank, nw, epoch,
                                        done);
  note_launch();
}

void launch_xcombine_sharded(char* own, const XLayout& L, uint32_t n, uint32_t epoch, bool reorder, uint8_t* status,
                             const uint8_t* lflag, const uint32_t* pmask, const uint32_t* grank, const uint8_t* ptype,
                             const uint8_t* params, long long* res, uint32_t rank, uint32_t nw, uint32_t* err,
                             uint32_t* err_all, cudaStream_t s) {
  // every block waits for the signals itself, so the grid is kept to one wave
  const uint32_t blocks = std::max<uint32_t>(1, std::min<uint32_t>((n + 255) / 256, 148 * 4));
  k_xcombine_sharded<<<blocks, 256, 0, s>>>(own, L, n, epoch, reorder, status, lflag, pmask, grank, ptype, params, res,
                                            rank, nw, err, err_all);
  note_launch();
}

void launch_xsig_res(const XPeers& peers, uint32_t rank, uint32_t world, uint32_t epoch, cudaStream_t s) {
  k_xsig_res<<<1, 64, 0, s>>>(peers, rank, world, epoch);
  note_launch();
}

void launch_xsum(const XPeers& peers, const XLayout& L, uint64_t n_reads, uint32_t epoch, long long* out,
                 uint32_t* err, uint32_t rank, uint32_t* done, cudaStream_t s) {
  // every block waits for the signals itself, so the grids are kept to one wave
  k_xrs<<<148 * 4, 256, 0, s>>>(peers, L, n_reads, epoch, err, rank, done);
  k_xag<<<148 * 4, 256, 0, s>>>(peers, L, n_reads, epoch, out, err, rank);
  note_launch(2);
}

}  // namespace ltpg
