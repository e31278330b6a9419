// C-ABI implementation (include/ltpg.h): device store management and the
// per-batch driver.  One ltpg_run_batch enqueues, on the caller's stream:
//   upload -> [per partition: K-group -> K-claim -> K-exec -> K-detect]
//   -> exchange (partitioned only: loopback OR / peer-memory stores between ranks)
//   -> [per partition: K-wb] -> finalize (commit bits, abort list) -> download
// The paper separates its three kernels with cudaDeviceSynchronize() (P:122,
// P:137-141); here stream order gives the same global isolation with no host
// round trip inside the batch.
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "ltpg_internal.cuh"
#include "tpcc_internal.cuh"
#include "xchg.cuh"

// NVTX ranges around the C-ABI calls (SURVEY §5 tracing): nsys timelines and `ncu --nvtx
// --nvtx-include "ltpg_run_batch/"` (header-only nvtx3: no cost without an attached tool)
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};


using namespace ltpg;

namespace {

uint64_t g_tab_versions = 0;
constexpr uint64_t LARGE_BUCKET_BYTES = 64ull << 20;  // NEXT-3 bucket memory cap per table     // process-wide: every table load gets a new version
uint64_t g_uploaded[64] = {0};   // per device: version whose tables sit in __constant__
// per device: recorded after every batch's device work (any db).  A db that re-uploads the
// constant bank (another db's tables were there) first waits on it, so the kernels of the
// previous owner -- possibly still running on another stream -- never see the new tables.
// the completion event (a slot's comp_done) of the last batch that ran with this device's
// constant bank, and its db: a db uploading other tables waits for it.  Not owned.
cudaEvent_t g_const_last[64] = {nullptr};
const void* g_const_owner[64] = {nullptr};

// per-partition scratch (one per logical partition handled by this process)
struct Part {
  long long* res = nullptr;
  unsigned long long* uref = nullptr;
  unsigned long long* items = nullptr;
  uint32_t* txn_ins = nullptr;
  uint8_t* ua = nullptr;
  uint8_t* lflag = nullptr;
  uint32_t* pmask = nullptr;             // sharded batches: partitions each shard txn touches
  uint32_t* small = nullptr;             // [0] err [1] ins_tables [2..7] kcount
  unsigned long long* base = nullptr;    // [MAXT]
  TpccDev tpcc;
};

// What a captured batch graph bakes in: every launch geometry and pointer of the batch's
// device work.  Two batches with equal keys enqueue identical work except for the BatchVars
// (epoch, clock), which the graph copies from the slot's pinned host copy when it runs.
struct GraphKey {
  uint32_t mode, n, n_ops, bflags, host_out, reads_dev, inputs_dev, packed;
  uint32_t small_w0, pad;  // single-launch kernel writes its result word 0 (no index catch-up ahead)
  uint64_t tab_version;
  const void* in[7];   // tid, op_begin, ops, args, ptype, params, offsets (device inputs only)
  const void* out[5];  // status, bits, abort, n_aborted, reads
  bool operator==(const GraphKey& o) const { return std::memcmp(this, &o, sizeof(*this)) == 0; }
};
struct GraphEntry {
  GraphKey key{};
  cudaGraphExec_t exec = nullptr;
  uint64_t launches = 0, last_use = 0;
};
constexpr int GRAPHS_PER_SLOT = 4;

// one in-flight batch: input staging, device outputs, pinned small results, events
struct Slot {
  unsigned long long* d_tid = nullptr;
  uint32_t* d_grank = nullptr;             // sharded batches: global ranks of the shard's txns
  uint32_t* d_op_begin = nullptr;
  ltpg_op* d_ops = nullptr;
  long long* d_args = nullptr;
  uint8_t* d_ptype = nullptr;
  uint8_t* d_params = nullptr;
  uint8_t* d_packed = nullptr;             // packed parameter blocks (proc_offsets)
  uint32_t* d_offsets = nullptr;
  long long* d_res = nullptr;              // combined results
  uint8_t* d_status = nullptr;
  uint32_t* d_bits = nullptr;
  uint32_t* d_flags = nullptr;
  uint32_t* d_offs = nullptr;
  uint32_t* d_abort = nullptr;
  uint32_t* d_small = nullptr;             // [0] err (combined) [8..10] counts
  uint32_t* h_small = nullptr;             // pinned + mapped: [0..15] d_small, [16] n_aborted
  uint32_t* h_small_dev = nullptr;         // its device-side address (written by k_publish)
  cudaEvent_t ev[8]{};
  cudaEvent_t h2d_done = nullptr, comp_done = nullptr, out_done = nullptr;
  cudaEvent_t out_ev = nullptr;  // the batch's last event: out_done, or comp_done when nothing follows it
  bool pending = false, timing = false, host_out = false, empty = false;
  ltpg_result* res = nullptr;
  uint64_t launches0 = 0;
  BatchVars* d_vars = nullptr;             // this batch's epoch / clock (read by the kernels)
  BatchVars* h_vars = nullptr;             // pinned + mapped host copy (read by graph replays)
  BatchVars* h_vars_dev = nullptr;         // its device-side address
  GraphEntry graphs[GRAPHS_PER_SLOT];
  // the batch's effective device inputs and abort list (LTPG_BATCH_CARRY_ABORTS of the next one)
  const unsigned long long* eff_tid = nullptr;
  const uint8_t* eff_ptype = nullptr;
  const uint8_t* eff_params = nullptr;
  const uint32_t* eff_abort = nullptr;
  uint64_t seq = 0;
  bool carry_src = false;  // a TPC-C batch of a single-rank db: its aborts can be carried
};

}  // namespace

struct ltpg_db {
  ltpg_config cfg{};
  int device = 0;
  bool poisoned = false;
  std::string last_error;
  uint32_t epoch = 0;
  uint32_t mark_window = 0;  // epoch / 255 of the last batch: a new window clears the marks
  uint32_t n_tables = 0;
  uint64_t tab_version = 0;
  uint32_t nparts = 1;     // global logical partitions = world * loopback
  uint32_t loopback = 1;   // partitions handled by this process
  DevTable h_tab[MAXT]{};
  DevTable* d_tab = nullptr;
  unsigned long long* d_nrows = nullptr;   // [MAXT]
  unsigned long long* d_reserve = nullptr; // [MAXT]
  uint32_t* d_dense_live = nullptr;        // bitmask: tables whose dense key->row mapping is valid
  bool olrow_ready = false;                // TPC-C ORDER -> first ORDER_LINE row map built
  bool tpcc_small_clean = false;           // partition 0's TPC-C batch scratch is in k_tpcc_small's
                                           // rest state (set by it; a multi-kernel batch clears it)
  // Deferred PK index maintenance: TPC-C reaches new ORDER_LINE rows through ORDER.aux only,
  // so their write-back skips the hash insert; rows >= d_idx_from[t] of a table in idx_lag
  // are indexed in one pass before anything else could look them up by key (an OPS batch,
  // the ORDER -> ORDER_LINE map rebuild).
  uint32_t idx_lag = 0;
  unsigned long long* d_idx_from = nullptr;  // [MAXT]
  uint16_t* d_su = nullptr;                  // [MAXT] NEXT-3: this batch's bucket size per table
  uint32_t* d_wprefix = nullptr;             // LTPG_RESULT_COMMITTED_READS: commits before each bitmask word
  uint32_t* d_coop = nullptr;                // [4096] per-block partial sums of cooperative kernels
  // LTPG_FLAG_L2_PERSIST_MARKS: the largest mark array (base, bytes) under an L2 persisting window
  void* persist_base = nullptr;
  size_t persist_bytes = 0;
  std::vector<Part> parts;
  void** d_ptrs = nullptr;                 // [3 * 64] partition pointer tables
  uint32_t* d_scan = nullptr;
  // inter-batch pipeline (NEXT-2): three slots, each with its own input staging and
  // output buffers, so batch n+1's H2D and batch n-1's D2H overlap batch n's kernels
  Slot slots[3];
  uint64_t submitted = 0;
  // LTPG_BATCH_CARRY_ABORTS: the last completed batch's conflict aborts, still on the device
  bool carry_ok = false;
  uint64_t carry_seq = 0;
  uint32_t carry_n = 0;
  int carry_slot = -1;
  cudaStream_t h2d = nullptr, d2h = nullptr;
  cudaStream_t cap = nullptr;              // batch graphs are captured here (never executes work)
  // batches execute in submission order even when the caller passes different streams:
  // each batch's first kernel waits on the previous batch's compute (they share scratch)
  uint64_t graph_uses = 0;
  // a8 (commit bitmask, abort list) runs on its own stream once the verdicts are final,
  // concurrently with write-back; it has its own scan scratch
  cudaStream_t fin = nullptr;
  cudaEvent_t status_ready = nullptr, fin_done = nullptr;
  uint32_t* d_scan_fin = nullptr;
  unsigned long long* d_fc_state = nullptr;  // a8 look-back tile states; [0] of d_fc_ctr: tile counter
  uint32_t* d_fc_ctr = nullptr;
  // peer-memory exchange between ranks (world > 1; xchg.cuh)
  bool p2p = false, connected = false;
  XLayout xl;
  XPeers xpeers{};
  char* xregion = nullptr;
  uint32_t* d_xdone = nullptr;              // [0] k_xput, [1] k_xrs block counters
  long long* d_xsink = nullptr;             // all-gather target when the caller wants no reads
  std::vector<void*> opened;  // peer regions mapped with cudaIpcOpenMemHandle
};

// what ltpg_peer_handle exports (LTPG_PEER_HANDLE_BYTES)
struct PeerHandle {
  cudaIpcMemHandle_t h;
  uint64_t bytes;
  uint32_t magic, rank, world, max_txns, max_ops, flags;
  uint8_t pad[LTPG_PEER_HANDLE_BYTES - sizeof(cudaIpcMemHandle_t) - 8 - 24];
};
static_assert(sizeof(PeerHandle) == LTPG_PEER_HANDLE_BYTES, "peer handle size");
constexpr uint32_t PEER_MAGIC = 0x4C545047u;  // "LTPG"

namespace {

int fail(ltpg_db* db, int code, const std::string& msg) {
  if (db) {
    db->last_error = msg;
    if (code == LTPG_ECUDA || code == LTPG_EINTERNAL) db->poisoned = true;
  }
  return code;
}

#define CK(call)                                                                          \
  do {                                                                                    \
    cudaError_t e_ = (call);                                                              \
    if (e_ != cudaSuccess)                                                                \
      return fail(db, e_ == cudaErrorMemoryAllocation ? LTPG_ENOMEM : LTPG_ECUDA,         \
                  std::string(#call) + ": " + cudaGetErrorString(e_));                   \
  } while (0)

template <class T>
cudaError_t dmalloc(T** p, size_t n) {
  return cudaMalloc(reinterpret_cast<void**>(p), std::max<size_t>(n, 1) * sizeof(T));
}

void free_table(DevTable& T) {
  if (T.dyn) cudaFree(T.dyn);
  if (T.stat) cudaFree(T.stat);
  if (T.valid) cudaFree(T.valid);
  if (T.rowkey) cudaFree(T.rowkey);
  if (T.wmarks) cudaFree(T.wmarks);
  if (T.amarks) cudaFree(T.amarks);
  if (T.rmarks) cudaFree(T.rmarks);
  if (T.idx) cudaFree(T.idx);
  if (T.aux) cudaFree(T.aux);
  for (mark_t* p : T.sub)
    if (p) cudaFree(p);
  unsigned long long* nr = T.n_rows;
  T = DevTable{};
  T.n_rows = nr;
}

// ---- exchange / combine kernels ------------------------------------------------------------
// A partition's verdict per txn is a set of conflict bits (CF_UA, CF_WAW, CF_RAW, CF_WAR); the
// txn's bits are the OR over partitions, then the commit rule applies (R1 or NEXT-1).
// loopback: OR in one kernel; the OR of all partitions' errors is written back to every
// partition so that none writes back.
__global__ void k_combine(void* const* lflags, uint32_t np, uint32_t n, uint8_t* status, void* const* errs,
                          uint32_t* err_all, bool reorder) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r == 0) {
    uint32_t e = 0;
    for (uint32_t p = 0; p < np; ++p) e |= *static_cast<const uint32_t*>(errs[p]);
    *err_all = e;
  }
  if (r >= n) return;
  uint32_t f = 0;
  for (uint32_t p = 0; p < np; ++p) f |= static_cast<const uint8_t*>(lflags[p])[r];
  status[r] = status_of_bits(f, reorder);
}
__global__ void k_spread_err(const uint32_t* err_all, void* const* errs, uint32_t np) {
  for (uint32_t p = 0; p < np; ++p) *static_cast<uint32_t*>(errs[p]) = *err_all;
}
__global__ void k_sum_res(void* const* res, uint32_t np, uint64_t n, long long* out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    unsigned long long s = 0;
    for (uint32_t p = 0; p < np; ++p) s += (unsigned long long)static_cast<const long long*>(res[p])[i];
    out[i] = (long long)s;
  }
}
__global__ void k_copy_err(const uint32_t* src, uint32_t* dst) { *dst = *src; }
// err_extra (single partition): the partition's own error word, ORed into word 0 here instead of
// a k_or_err launch at the end of every batch
__global__ void k_publish(const uint32_t* src, volatile uint32_t* host_dst, uint32_t n, const uint32_t* err_extra) {
  if (threadIdx.x < n) host_dst[threadIdx.x] = src[threadIdx.x] | (threadIdx.x == 0 && err_extra ? *err_extra : 0u);
}
// batch start: append reservations cleared and the batch scalars stored where the kernels read
// them -- from the arguments (direct enqueue) or, in a replayed graph, from the slot's pinned
// host copy through its mapped address (read when the graph runs, not when it was captured)
// + partition 0's small words (error, counters) and user-abort flags, which were two memset
// nodes of their own ahead of every batch
__global__ void k_batch_init(unsigned long long* reserve, BatchVars* vars, const volatile BatchVars* host,
                             uint32_t epoch, long long clock, uint32_t* small0, uint8_t* ua0, uint32_t n,
                             uint32_t* tmisc, uint32_t* dl_min, uint32_t nw) {
  if (blockIdx.x == 0) {
    if (threadIdx.x < MAXT) reserve[threadIdx.x] = 0;
    if (threadIdx.x < 16) small0[threadIdx.x] = 0;
    if (tmisc) {  // TPC-C partition 0: batch counters, smallest Delivery rank per warehouse (none)
      if (threadIdx.x < 16) tmisc[threadIdx.x] = 0;
      for (uint32_t w = threadIdx.x; w <= nw; w += blockDim.x) dl_min[w] = ~0u;
    }
    if (threadIdx.x == 0) {
      vars->epoch = host ? host->epoch : epoch;
      vars->clock = host ? host->clock : clock;
    }
  }
  const uint32_t n16 = n / 16;  // ua0 is 256-byte aligned (cudaMalloc)
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += gridDim.x * blockDim.x)
    reinterpret_cast<uint4*>(ua0)[i] = make_uint4(0, 0, 0, 0);
  if (blockIdx.x == 0 && threadIdx.x < n % 16) ua0[16 * n16 + threadIdx.x] = 0;
}
__global__ void k_or_err(const uint32_t* src, uint32_t* dst) {
  if (*src) *dst |= *src;
}

}  // namespace

extern "C" {

const char* ltpg_version(void) { return "ltpg-b200 0.2 sm_100a"; }

const char* ltpg_last_error(const ltpg_db* db) { return db ? db->last_error.c_str() : "null db"; }

int ltpg_create_db(const ltpg_config* cfg, ltpg_db** out) {
  ltpg_db* db = nullptr;
  if (!cfg || !out) return LTPG_EINVAL;
  const uint32_t loop = std::max<uint32_t>(1, (cfg->flags >> LTPG_FLAG_LOOPBACK_SHIFT) & 0xF);
  if (cfg->n_tables == 0 || cfg->n_tables > MAXT || cfg->max_txns == 0 || cfg->world < 1 ||
      cfg->rank < 0 || cfg->rank >= cfg->world || cfg->max_txns > (1u << 24) || cfg->max_ops > (1u << 24) ||
      cfg->n_warehouses > 1000 || cfg->world * loop > 64 || cfg->world > 32 || (cfg->flags & LTPG_FLAG_RESERVED_4) ||
      (cfg->world > 1 && loop > 1))
    return LTPG_EINVAL;
  db = new ltpg_db();
  db->cfg = *cfg;
  db->device = cfg->device;
  db->n_tables = cfg->n_tables;
  db->loopback = loop;
  db->nparts = (uint32_t)cfg->world * loop;
  *out = db;
  CK(cudaSetDevice(cfg->device));
  const size_t n = cfg->max_txns, m = std::max<uint32_t>(cfg->max_ops, 1);
  const size_t nres = std::max(m, n * LTPG_PROC_RESULTS);
  CK(dmalloc(&db->d_tab, MAXT));
  CK(dmalloc(&db->d_nrows, MAXT));
  CK(cudaMemset(db->d_nrows, 0, MAXT * sizeof(unsigned long long)));
  CK(dmalloc(&db->d_reserve, MAXT));
  CK(dmalloc(&db->d_idx_from, MAXT));
  CK(dmalloc(&db->d_su, MAXT));
  CK(dmalloc(&db->d_wprefix, (n + 31) / 32 + 1));
  CK(dmalloc(&db->d_coop, 4096));
  CK(cudaMemset(db->d_su, 0, MAXT * sizeof(uint16_t)));
  CK(dmalloc(&db->d_dense_live, 1));
  CK(cudaMemset(db->d_dense_live, 0, sizeof(uint32_t)));
  for (int t = 0; t < MAXT; ++t) db->h_tab[t].n_rows = db->d_nrows + t;
  for (Slot& S : db->slots) {
    CK(dmalloc(&S.d_tid, n));
    CK(dmalloc(&S.d_grank, n));
    CK(dmalloc(&S.d_op_begin, n + 1));
    CK(dmalloc(&S.d_ops, m));
    CK(dmalloc(&S.d_args, m));
    CK(dmalloc(&S.d_ptype, n));
    CK(dmalloc(&S.d_params, n * LTPG_PARAM_BYTES));
    CK(dmalloc(&S.d_packed, n * LTPG_PARAM_BYTES));
    CK(dmalloc(&S.d_offsets, n + 1));
    CK(dmalloc(&S.d_res, nres));
    CK(dmalloc(&S.d_status, n));
    CK(dmalloc(&S.d_bits, (n + 31) / 32 + 1));
    CK(dmalloc(&S.d_flags, n));
    CK(dmalloc(&S.d_offs, n + 1));
    CK(dmalloc(&S.d_abort, n));
    CK(dmalloc(&S.d_small, 64));
    CK(cudaHostAlloc(reinterpret_cast<void**>(&S.h_small), 64 * sizeof(uint32_t), cudaHostAllocMapped));
    CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&S.h_small_dev), S.h_small, 0));
    for (auto& e : S.ev) CK(cudaEventCreate(&e));
    CK(cudaEventCreateWithFlags(&S.h2d_done, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&S.comp_done, cudaEventDisableTiming));
    CK(cudaEventCreate(&S.out_done));  // (timed: ltpg_stats.ms_download)
    S.out_ev = S.out_done;
    CK(dmalloc(&S.d_vars, 1));
    CK(cudaHostAlloc(reinterpret_cast<void**>(&S.h_vars), sizeof(BatchVars), cudaHostAllocMapped));
    CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&S.h_vars_dev), S.h_vars, 0));
  }
  CK(dmalloc(&db->d_ptrs, 3 * 64));
  CK(dmalloc(&db->d_scan, scan_scratch_words(std::max<size_t>(n, m)) + 16));
  CK(cudaStreamCreateWithFlags(&db->h2d, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&db->d2h, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&db->fin, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&db->cap, cudaStreamNonBlocking));
  CK(cudaEventCreateWithFlags(&db->status_ready, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&db->fin_done, cudaEventDisableTiming));
  CK(dmalloc(&db->d_scan_fin, scan_scratch_words(n) + 16));
  CK(dmalloc(&db->d_fc_state, (n + 1023) / 1024 + 1));
  CK(cudaMemset(db->d_fc_state, 0, ((n + 1023) / 1024 + 1) * sizeof(unsigned long long)));
  CK(dmalloc(&db->d_fc_ctr, 1));
  CK(cudaMemcpy(db->d_tab, db->h_tab, sizeof(db->h_tab), cudaMemcpyHostToDevice));
  db->parts.resize(loop);
  std::vector<void*> ptrs(3 * 64, nullptr);
  for (uint32_t p = 0; p < loop; ++p) {
    Part& P = db->parts[p];
    CK(dmalloc(&P.res, nres));
    CK(dmalloc(&P.uref, m));
    CK(dmalloc(&P.items, m * NKINDS));
    CK(dmalloc(&P.txn_ins, n + 1));
    CK(dmalloc(&P.ua, n));
    CK(dmalloc(&P.lflag, n + 4));  // (k_ops_small ORs verdict bytes as 32-bit words)
    CK(dmalloc(&P.pmask, n));
    // [0, 16) the partition's words; [16, 64) per-slot sets (single-launch kernels); [64 + 32 k]
    // slot k's grid-barrier counter (one 128-byte line each)
    CK(dmalloc(&P.small, 64 + 3 * 32));
    CK(cudaMemset(P.small, 0, (64 + 3 * 32) * sizeof(uint32_t)));
    CK(dmalloc(&P.base, MAXT));
    int rc = tpcc_alloc(P.tpcc, cfg->max_txns, cfg->n_warehouses, p ? db->parts[0].tpcc.by_name : nullptr);
    if (rc) return fail(db, rc, "tpcc scratch allocation failed (n_warehouses <= 1000)");
    P.tpcc.h_tab = db->h_tab;
    P.tpcc.n_tab = cfg->n_tables;
    P.tpcc.d_su = db->d_su;
    ptrs[p] = P.lflag;
    ptrs[64 + p] = P.small;
    ptrs[128 + p] = P.res;
  }
  CK(cudaMemcpy(db->d_ptrs, ptrs.data(), ptrs.size() * sizeof(void*), cudaMemcpyHostToDevice));
  if (cfg->world > 1) {  // peer-memory exchange region
    db->p2p = true;
    db->xl.init(cfg->max_txns, nres, (uint32_t)cfg->world);
    CK(cudaMalloc(reinterpret_cast<void**>(&db->xregion), db->xl.bytes));
    CK(cudaMemset(db->xregion, 0, db->xl.bytes));
    CK(dmalloc(&db->d_xdone, 2));
    CK(cudaMemset(db->d_xdone, 0, 2 * sizeof(uint32_t)));
    CK(dmalloc(&db->d_xsink, nres));
    db->xpeers.base[cfg->rank] = db->xregion;
  }
  return LTPG_OK;
}

void ltpg_destroy_db(ltpg_db* db) {
  if (!db) return;
  cudaSetDevice(db->device);
  cudaDeviceSynchronize();
  for (int t = 0; t < MAXT; ++t) free_table(db->h_tab[t]);
  void* bufs[] = {db->d_tab, db->d_nrows, db->d_reserve, db->d_dense_live, db->d_ptrs, db->d_scan,
                  db->d_idx_from, db->d_su, db->d_wprefix, db->d_coop};
  for (void* p : bufs)
    if (p) cudaFree(p);
  for (Slot& S : db->slots) {
    void* sb[] = {S.d_tid, S.d_grank, S.d_op_begin, S.d_ops, S.d_args, S.d_ptype, S.d_params, S.d_packed, S.d_offsets,
                  S.d_res, S.d_status,
                  S.d_bits, S.d_flags, S.d_offs, S.d_abort, S.d_small, S.d_vars};
    for (void* p : sb)
      if (p) cudaFree(p);
    if (S.h_small) cudaFreeHost(S.h_small);
    if (S.h_vars) cudaFreeHost(S.h_vars);
    for (GraphEntry& g : S.graphs)
      if (g.exec) cudaGraphExecDestroy(g.exec);
    for (auto& e : S.ev)
      if (e) cudaEventDestroy(e);
    for (cudaEvent_t e : {S.h2d_done, S.comp_done, S.out_done})
      if (e) cudaEventDestroy(e);
  }
  if (db->h2d) cudaStreamDestroy(db->h2d);
  if (db->d2h) cudaStreamDestroy(db->d2h);
  if (db->fin) cudaStreamDestroy(db->fin);
  if (db->cap) cudaStreamDestroy(db->cap);
  if (db->status_ready) cudaEventDestroy(db->status_ready);
  if (db->fin_done) cudaEventDestroy(db->fin_done);
  if (g_const_owner[db->device % 64] == db) {  // (cudaFree below synchronizes the device)
    g_const_last[db->device % 64] = nullptr;
    g_const_owner[db->device % 64] = nullptr;
  }
  if (db->d_scan_fin) cudaFree(db->d_scan_fin);
  if (db->d_fc_state) cudaFree(db->d_fc_state);
  if (db->d_fc_ctr) cudaFree(db->d_fc_ctr);
  for (Part& P : db->parts) {
    void* pb[] = {P.res, P.uref, P.items, P.txn_ins, P.ua, P.lflag, P.pmask, P.small, P.base};
    for (void* p : pb)
      if (p) cudaFree(p);
    tpcc_free(P.tpcc);
  }
  for (void* p : db->opened) cudaIpcCloseMemHandle(p);
  if (db->xregion) cudaFree(db->xregion);
  if (db->d_xdone) cudaFree(db->d_xdone);
  if (db->d_xsink) cudaFree(db->d_xsink);
  delete db;
}

int ltpg_load_table(ltpg_db* db, uint32_t t, const ltpg_table_desc* d, uint64_t n_rows, const uint64_t* keys,
                    const int64_t* cols) {
  if (!db) return LTPG_EINVAL;
  NvtxRange nvtx_range("ltpg_load_table");
  if (db->poisoned) return LTPG_EPOISONED;
  if (!d || t >= db->n_tables || d->n_cols > MAXC || (d->n_cols && (!d->col_group || !d->col_is_add)) ||
      n_rows > d->capacity_rows || d->capacity_rows >= 0xFFFFFFF0ull || (n_rows && d->n_cols && !cols) ||
      (d->has_pk && n_rows && !keys) || d->n_groups > 15 || d->owner_rule > 2 || d->layout > LTPG_LAYOUT_COLUMNAR)
    return fail(db, LTPG_EINVAL, "bad table descriptor");
  bool has_static = false;
  for (uint32_t c = 0; c < d->n_cols; ++c) {
    uint8_t g = d->col_group[c];
    if (g == LTPG_STATIC) {
      has_static = true;
      if (d->col_is_add[c]) return fail(db, LTPG_EINVAL, "static ADD column");
    } else if (g >= d->n_groups) {
      return fail(db, LTPG_EINVAL, "column group out of range");
    }
    for (uint32_t e = 0; e < d->n_cols; ++e)  // an ADD group holds ADD columns only
      if (g != LTPG_STATIC && d->col_group[e] == g && (d->col_is_add[e] != 0) != (d->col_is_add[c] != 0))
        return fail(db, LTPG_EINVAL, "mixed ADD / plain column group");
  }
  CK(cudaSetDevice(db->device));
  CK(cudaDeviceSynchronize());
  DevTable& T = db->h_tab[t];
  if (T.wmarks && T.wmarks == db->persist_base) {  // its marks go away: no window over freed memory
    db->persist_base = nullptr;
    db->persist_bytes = 0;
  }
  free_table(T);
  const uint64_t cap = std::max<uint64_t>(d->capacity_rows, 1);
  T.n_cols = d->n_cols;
  T.n_groups = d->n_groups;
  T.has_pk = d->has_pk ? 1 : 0;
  T.has_static = has_static;
  T.defined = 1;
  T.owner_rule = d->owner_rule;
  T.capacity = cap;
  T.id = t;
  // row-block layout: mutable block (non-static columns), static block; marks separate
  uint32_t n_dyn = 0, n_stat = 0;
  for (uint32_t c = 0; c < d->n_cols; ++c) (d->col_group[c] == LTPG_STATIC ? n_stat : n_dyn)++;
  // pad blocks of up to 8 words to a power of two (a row never straddles a 64 B unit); wider
  // rows stay unpadded so that appends from consecutive lanes fill whole sectors
  auto pad_words = [](uint32_t w) -> uint32_t {
    if (w == 0 || w > 8) return w;
    uint32_t p = 1;
    while (p < w) p <<= 1;
    return p;
  };
  T.dstride = pad_words(n_dyn);
  T.sstride = pad_words(n_stat);
  if (T.dstride) CK(dmalloc(&T.dyn, cap * T.dstride));
  if (T.sstride) CK(dmalloc(&T.stat, cap * T.sstride));
  T.group_bits = ~0ull;
  T.add_bits = 0;
  T.dyn_mask = 0;
  for (uint32_t c = 0, jd = 0, js = 0; c < d->n_cols; ++c) {
    const bool st = d->col_group[c] == LTPG_STATIC;
    T.col[c] = st ? T.stat + js++ : T.dyn + jd++;
    T.stride[c] = st ? T.sstride : T.dstride;
    T.group[c] = d->col_group[c];
    T.is_add[c] = d->col_is_add[c] ? 1 : 0;
    const uint64_t g = st ? 15u : d->col_group[c];
    T.group_bits = (T.group_bits & ~(15ull << (4 * c))) | (g << (4 * c));
    if (d->col_is_add[c]) T.add_bits |= 1u << c;
    if (!st) T.dyn_mask |= 1u << c;
  }
  if (d->layout == LTPG_LAYOUT_COLUMNAR) {
    if (T.dyn) cudaFree(T.dyn);
    if (T.stat) cudaFree(T.stat);
    T.dyn = T.stat = nullptr;
    T.columnar = 1;
    T.dstride = T.sstride = 1;
    CK(dmalloc(&T.dyn, cap * std::max<uint32_t>(d->n_cols, 1)));
    for (uint32_t c = 0; c < d->n_cols; ++c) {
      T.col[c] = T.dyn + c * cap;
      T.stride[c] = 1;
    }
  }
  CK(dmalloc(&T.valid, cap));
  CK(cudaMemset(T.valid, 0, cap));
  CK(dmalloc(&T.rowkey, cap));
  if (d->n_groups) {  // every mark starts "unmarked" (0xFF tag byte: no live epoch)
    T.add_groups = 0;
    for (uint32_t c = 0; c < d->n_cols; ++c)
      if (d->col_is_add[c] && d->col_group[c] != LTPG_STATIC) T.add_groups |= 1u << d->col_group[c];
    CK(dmalloc(&T.wmarks, cap * d->n_groups));
    CK(cudaMemset(T.wmarks, 0xFF, cap * d->n_groups * sizeof(mark_t)));
    if ((db->cfg.flags & LTPG_FLAG_L2_PERSIST_MARKS) && cap * d->n_groups * sizeof(mark_t) > db->persist_bytes) {
      db->persist_base = T.wmarks;  // (a table reloaded later keeps the old pointer: refreshed below)
      db->persist_bytes = cap * d->n_groups * sizeof(mark_t);
    }
    if (const uint32_t na = __builtin_popcount(T.add_groups)) {
      CK(dmalloc(&T.amarks, cap * na));
      CK(cudaMemset(T.amarks, 0xFF, cap * na * sizeof(mark_t)));
    }
    if (db->cfg.flags & LTPG_FLAG_REORDER) {  // NEXT-1: minimum reader rank per unit
      CK(dmalloc(&T.rmarks, cap * d->n_groups));
      CK(cudaMemset(T.rmarks, 0xFF, cap * d->n_groups * sizeof(mark_t)));
    }
    // NEXT-3: a popular table -- E = T/D > 1 with T bounded by the batch capacity
    // and D the loaded rows -- gets large-sized buckets of su = ceil(E/32)*32 sub-slots for each
    // unit of its loaded rows (appended rows keep standard slots).  Buckets are only for
    // "limited" popular data: a table whose buckets would exceed LARGE_BUCKET_BYTES
    // stays standard-sized.
    const double E = (double)db->cfg.max_txns / (double)std::max<uint64_t>(n_rows, 1);
    const uint32_t na = __builtin_popcount(T.add_groups);
    if ((db->cfg.flags & LTPG_FLAG_LARGE_BUCKETS) && E > 1.0 && n_rows) {
      const uint64_t su = (uint64_t)std::ceil(E / 32.0) * 32;
      const uint64_t units[3] = {n_rows * d->n_groups, n_rows * na, T.rmarks ? n_rows * d->n_groups : 0};
      if ((units[0] + units[1] + units[2]) * su * sizeof(mark_t) <= LARGE_BUCKET_BYTES) {
        T.su = (uint32_t)su;
        T.sub_rows = (uint32_t)n_rows;
        for (int k = 0; k < 3; ++k) {
          if (!units[k]) continue;
          CK(dmalloc(&T.sub[k], units[k] * su));
          CK(cudaMemset(T.sub[k], 0xFF, units[k] * su * sizeof(mark_t)));
        }
      }
    }
  }
  if (d->has_pk) {
    uint64_t sz = 1;
    uint32_t bits = 0;
    while (sz < 2 * cap) sz <<= 1, ++bits;
    if (bits < 4) sz = 16, bits = 4;
    CK(dmalloc(&T.idx, sz));
    CK(cudaMemset(T.idx, 0xFF, sz * sizeof(IdxSlot)));
    T.idx_mask = sz - 1;
    T.idx_shift = 64 - bits;
  }
  if (n_rows) {
    long long* tmp = nullptr;  // column-major upload, scattered into the row blocks on the device
    if (d->n_cols) CK(dmalloc(&tmp, n_rows));
    for (uint32_t c = 0; c < d->n_cols; ++c) {
      CK(cudaMemcpy(tmp, cols + c * n_rows, n_rows * sizeof(int64_t), cudaMemcpyHostToDevice));
      launch_scatter_col(T.col[c], T.stride[c], tmp, n_rows, 0);
    }
    CK(cudaDeviceSynchronize());
    if (tmp) cudaFree(tmp);
    CK(cudaMemset(T.valid, 1, n_rows));
    if (d->has_pk) CK(cudaMemcpy(T.rowkey, keys, n_rows * sizeof(uint64_t), cudaMemcpyHostToDevice));
  }
  // dense key range: keys[r] == keys[0] + r for every loaded row
  bool dense = d->has_pk && n_rows > 0;
  for (uint64_t r = 1; dense && r < n_rows; ++r) dense = keys[r] == keys[0] + r;
  T.key_base = dense ? keys[0] : 0;
  T.dense_n = dense ? n_rows : 0;
  uint32_t live = 0;
  CK(cudaMemcpy(&live, db->d_dense_live, sizeof(live), cudaMemcpyDeviceToHost));
  live = dense ? (live | (1u << t)) : (live & ~(1u << t));
  CK(cudaMemcpy(db->d_dense_live, &live, sizeof(live), cudaMemcpyHostToDevice));
  if (t == LTPG_T_ORDER && db->cfg.n_warehouses) {
    CK(dmalloc(&T.aux, cap));
    CK(cudaMemset(T.aux, 0xFF, cap * sizeof(uint32_t)));
  }
  if (t == LTPG_T_ORDER || t == LTPG_T_ORDER_LINE) db->olrow_ready = false;
  db->idx_lag &= ~(1u << t);  // the index is rebuilt from every loaded row below
  unsigned long long nr = n_rows;
  CK(cudaMemcpy(T.n_rows, &nr, sizeof(nr), cudaMemcpyHostToDevice));
  CK(cudaMemcpy(db->d_tab, db->h_tab, sizeof(db->h_tab), cudaMemcpyHostToDevice));
  db->tab_version = ++g_tab_versions;
  if (d->has_pk && n_rows) {
    uint32_t* d_err = db->slots[0].d_small;
    CK(cudaMemset(d_err, 0, sizeof(uint32_t)));
    upload_tables_common(db->d_tab, 0);
    g_uploaded[db->device % 64] = 0;
    launch_build_index(t, 0, n_rows, d_err, 0);
    CK(cudaGetLastError());
    uint32_t err = 0;
    CK(cudaMemcpy(&err, d_err, sizeof(err), cudaMemcpyDeviceToHost));
    if (err) {
      free_table(T);
      cudaMemcpy(db->d_tab, db->h_tab, sizeof(db->h_tab), cudaMemcpyHostToDevice);
      return fail(db, LTPG_EINVAL, "duplicate or reserved primary key");
    }
  }
  if (t == LTPG_T_CUSTOMER && db->cfg.n_warehouses && !db->parts.empty()) {
    int rc = tpcc_build_secondary(db->parts[0].tpcc, keys, cols, n_rows, db->cfg.n_warehouses);
    if (rc) return fail(db, rc, "secondary index build failed");
  }
  CK(cudaDeviceSynchronize());
  return LTPG_OK;
}

}  // extern "C"

namespace {

// Complete the batch held by slot S: wait for its outputs, report errors / counts / stages.
int finish_slot(ltpg_db* db, Slot& S) {
  S.pending = false;
  db->carry_ok = false;
  CK(cudaEventSynchronize(S.out_ev));
  const uint32_t err = S.h_small[0];
  if (err & ERR_EINTERNAL) return fail(db, LTPG_EINTERNAL, "device invariant violated");
  if (err & ERR_EINVAL) return fail(db, LTPG_EINVAL, "invalid batch (validated on device; nothing changed)");
  if (err & ERR_ECAPACITY) return fail(db, LTPG_ECAPACITY, "append capacity exceeded (nothing changed)");
  if (S.host_out) *S.res->n_aborted = S.h_small[16];
  if (S.carry_src) {  // its conflict aborts can lead the next batch (LTPG_BATCH_CARRY_ABORTS)
    db->carry_ok = true;
    db->carry_seq = S.seq;
    db->carry_n = S.h_small[16];
    db->carry_slot = (int)(&S - db->slots);
  }
  if (S.timing && S.empty) {  // nothing ran: no stage events were recorded
    *S.res->stats = ltpg_stats{};
  } else if (S.timing) {
    ltpg_stats* st = S.res->stats;
    float ms[7] = {0};
    for (int i = 0; i < 6; ++i) CK(cudaEventElapsedTime(&ms[i], S.ev[i], S.ev[i + 1]));
    CK(cudaEventElapsedTime(&ms[6], S.ev[6], S.out_done));
    st->ms_upload = ms[0];
    st->ms_group = ms[1];
    st->ms_exec = ms[2];
    st->ms_detect = ms[3];
    st->ms_exchange = ms[4];
    st->ms_writeback = ms[5];
    st->ms_download = ms[6];
    st->n_commit = S.h_small[8];
    st->n_conflict = S.h_small[9];
    st->n_user_abort = S.h_small[10];
    st->popular_tables = S.h_small[11];
  }
  return LTPG_OK;
}

}  // namespace

extern "C" {

int ltpg_pending_aborts(ltpg_db* db, uint32_t* n) {
  if (!db || !n) return LTPG_EINVAL;
  *n = (db->carry_ok && db->carry_seq == db->submitted) ? db->carry_n : 0u;
  return LTPG_OK;
}

int ltpg_wait_batch(ltpg_db* db, ltpg_result* res) {
  if (!db || !res) return LTPG_EINVAL;
  NvtxRange nvtx_range("ltpg_wait_batch");
  for (Slot& S : db->slots)
    if (S.pending && S.res == res) return finish_slot(db, S);
  return fail(db, LTPG_EINVAL, "no batch in flight for this result");
}

int ltpg_run_batch(ltpg_db* db, const ltpg_batch* b, ltpg_result* res) {
  if (!db) return LTPG_EINVAL;
  NvtxRange nvtx_range("ltpg_run_batch");
  if (db->poisoned) return LTPG_EPOISONED;
  if (!b || !res || !b->tid || !res->commit_bits || !res->n_aborted ||
      (!res->status && !(res->flags & LTPG_RESULT_NO_STATUS)) ||
      (!res->abort_idx && !(res->flags & LTPG_RESULT_NO_ABORT_LIST)))
    return fail(db, LTPG_EINVAL, "null argument");
  const uint32_t nf = b->n_txns;  // txns given (LTPG_BATCH_CARRY_ABORTS: after the carried ones)
  const bool ops_mode = b->mode == LTPG_MODE_OPS;
  const bool carry = (b->flags & LTPG_BATCH_CARRY_ABORTS) != 0;
  if (carry && (ops_mode || b->inputs_on_device || db->cfg.world > 1 || (db->cfg.flags & LTPG_FLAG_GRAPH) ||
                !db->carry_ok || db->carry_seq != db->submitted))
    return fail(db, LTPG_EINVAL, "LTPG_BATCH_CARRY_ABORTS: TPCC host inputs on a single-rank, non-graph db, after "
                                 "the previous batch completed");
  const bool tid_range = (b->flags & LTPG_BATCH_TID_RANGE) != 0;
  if (tid_range && b->inputs_on_device) return fail(db, LTPG_EINVAL, "LTPG_BATCH_TID_RANGE: host inputs only");
  const unsigned long long tid0 = tid_range && nf ? (unsigned long long)b->tid[0] : 0ull;
  const uint32_t nc = carry ? db->carry_n : 0u;  // carried conflict aborts of the previous batch
  const uint32_t n = nc + nf;
  if ((uint64_t)nc + nf > db->cfg.max_txns) return fail(db, LTPG_EINVAL, "n_txns > max_txns"); 
  if (!ops_mode && b->mode != LTPG_MODE_TPCC) return fail(db, LTPG_EINVAL, "bad mode");
  if (ops_mode && (b->n_ops > db->cfg.max_ops || !b->op_begin || (b->n_ops && (!b->ops || !b->op_arg))))
    return fail(db, LTPG_EINVAL, "bad OPS batch");
  if (!ops_mode && (!b->proc_type || !b->proc_params || !db->cfg.n_warehouses))
    return fail(db, LTPG_EINVAL, "bad TPCC batch");
  if ((b->flags & LTPG_BATCH_COMPACT_PARAMS) && (ops_mode || !b->proc_offsets))
    return fail(db, LTPG_EINVAL, "LTPG_BATCH_COMPACT_PARAMS needs a TPCC batch with proc_offsets");
  if (db->p2p && !db->connected) return fail(db, LTPG_EINVAL, "world > 1: ltpg_connect_peers first");
  if (!ops_mode && b->proc_offsets && !b->inputs_on_device && b->proc_offsets[nf] > (uint64_t)nf * LTPG_PARAM_BYTES)
    return fail(db, LTPG_EINVAL, "packed params too large");
  if (res->reads && res->reads_cap &&
      res->reads_cap < (ops_mode ? (uint64_t)b->n_ops : (uint64_t)n * LTPG_PROC_RESULTS))
    return fail(db, LTPG_EINVAL, "reads buffer smaller than the batch's result slots (reads_cap)");
  // LTPG_RESULT_COMMITTED_READS: the gather kernel writes the caller's buffer directly
  const bool cr = (res->flags & LTPG_RESULT_COMMITTED_READS) != 0;
  long long* cr_dst = nullptr;
  if (cr) {
    if (ops_mode || !res->reads) return fail(db, LTPG_EINVAL, "LTPG_RESULT_COMMITTED_READS: TPCC with a reads buffer");
    if (res->outputs_on_device) {
      cr_dst = reinterpret_cast<long long*>(res->reads);
    } else {
      cudaPointerAttributes pa{};
      if (cudaPointerGetAttributes(&pa, res->reads) != cudaSuccess || pa.type != cudaMemoryTypeHost ||
          !pa.devicePointer) {
        cudaGetLastError();
        return fail(db, LTPG_EINVAL, "LTPG_RESULT_COMMITTED_READS: the host reads buffer must be pinned and mapped");
      }
      cr_dst = static_cast<long long*>(pa.devicePointer);
    }
  }
  const bool sharded = b->grank != nullptr;
  if (sharded && (ops_mode || !db->p2p || b->n_global > db->cfg.max_txns || n > b->n_global))
    return fail(db, LTPG_EINVAL, "sharded batches: TPCC on a multi-rank peer-memory db, n_txns <= n_global <= max_txns");
  // every host-side validation is above this line: from here on the batch is submitted
  Slot& S = db->slots[db->submitted % 3];
  if (S.pending) return fail(db, LTPG_EINVAL, "three batches already in flight: ltpg_wait_batch first");
  ++db->submitted;
  CK(cudaSetDevice(db->device));
  cudaStream_t s = static_cast<cudaStream_t>(b->stream);
  const bool async = (b->flags & LTPG_BATCH_ASYNC) != 0;
  const bool timing = res->stats != nullptr;
  const bool partitioned = db->nparts > 1;
  const uint32_t L = db->loopback;
  const bool grouped = !(db->cfg.flags & LTPG_FLAG_NO_GROUPING);
  // small single-partition batches: a1..a8 in one cooperative launch (k_ops_small, k_tpcc_small),
  // with the slot's own set of partition small words (published and cleared by the kernel's last
  // block)
  const bool small = (ops_mode ? grouped && n <= ops_small_max_txns()
                               : n <= tpcc_small_max_txns() && tpcc_small_fits(db->parts[0].tpcc)) &&
                     L == 1 && !partitioned && !db->p2p && n &&
                     !(db->cfg.flags & (LTPG_FLAG_LARGE_BUCKETS | LTPG_FLAG_NO_SINGLE_LAUNCH));
  uint32_t* small_words = small ? db->parts[0].small + 16 * (1 + (&S - db->slots)) : nullptr;
  uint32_t* small_bar = small ? db->parts[0].small + 64 + 32 * (&S - db->slots) : nullptr;
  S.timing = timing;
  S.res = res;
  S.host_out = !res->outputs_on_device;
  S.launches0 = g_kernel_launches;
  S.empty = n == 0;
  ++db->epoch;
  // ---- a1: upload on the copy stream (overlaps the previous batch's kernels) ------------------
  BatchDev bd{};
  bd.nparts = db->nparts;
  bd.nw = db->cfg.n_warehouses;
  bd.key_space = db->cfg.key_space;
  bd.reserve = db->d_reserve;
  bd.dense_live = db->d_dense_live;
  bd.n_txns = n;
  bd.n_ops = ops_mode ? b->n_ops : 0;
  bd.flags = db->cfg.flags;
  bd.vars = S.d_vars;
  bd.max_ops = std::max<uint32_t>(db->cfg.max_ops, 1);
  bd.n_global = sharded ? b->n_global : n;
  // verdict outputs: written in place when the caller's buffers are on the device
  uint8_t* st_out = (S.host_out || !res->status) ? S.d_status : res->status;
  uint32_t* bits_out = S.host_out ? S.d_bits : res->commit_bits;
  uint32_t* abort_out = (S.host_out || !res->abort_idx) ? S.d_abort : res->abort_idx;
  bd.status = st_out;
  const cudaMemcpyKind h2d = cudaMemcpyHostToDevice;
  if (b->inputs_on_device) {
    bd.grank = b->grank;
    bd.tid = reinterpret_cast<const unsigned long long*>(b->tid);
    bd.op_begin = b->op_begin;
    bd.ops = b->ops;
    bd.args = reinterpret_cast<const long long*>(b->op_arg);
    bd.ptype = b->proc_type;
    bd.params = b->proc_params;
  } else {
    // the slot's staging buffers are free once its previous batch's kernels are done
    CK(cudaStreamWaitEvent(db->h2d, S.comp_done, 0));
    // (carried txns: positions [0, nc) are filled on the device by k_carry; the given ones follow)
    if (!tid_range) CK(cudaMemcpyAsync(S.d_tid + nc, b->tid, nf * sizeof(uint64_t), h2d, db->h2d));
    bd.tid = S.d_tid;
    if (sharded) {
      CK(cudaMemcpyAsync(S.d_grank, b->grank, n * sizeof(uint32_t), h2d, db->h2d));
      bd.grank = S.d_grank;
    }
    if (ops_mode) {
      CK(cudaMemcpyAsync(S.d_op_begin, b->op_begin, (n + 1) * sizeof(uint32_t), h2d, db->h2d));
      if (b->n_ops) {
        CK(cudaMemcpyAsync(S.d_ops, b->ops, b->n_ops * sizeof(ltpg_op), h2d, db->h2d));
        CK(cudaMemcpyAsync(S.d_args, b->op_arg, b->n_ops * sizeof(int64_t), h2d, db->h2d));
      }
      bd.op_begin = S.d_op_begin;
      bd.ops = S.d_ops;
      bd.args = S.d_args;
    } else {
      CK(cudaMemcpyAsync(S.d_ptype + nc, b->proc_type, nf, h2d, db->h2d));
      if (b->proc_offsets) {  // packed blocks: offsets + used bytes only, expanded on the GPU
        const uint64_t packed = b->proc_offsets[nf];  // <= nf * 128 (checked before submission)
        CK(cudaMemcpyAsync(S.d_offsets, b->proc_offsets, (nf + 1) * sizeof(uint32_t), h2d, db->h2d));
        CK(cudaMemcpyAsync(S.d_packed, b->proc_params, packed, h2d, db->h2d));
      } else {
        CK(cudaMemcpyAsync(S.d_params + (size_t)nc * LTPG_PARAM_BYTES, b->proc_params, (size_t)nf * LTPG_PARAM_BYTES,
                           h2d, db->h2d));
      }
      bd.ptype = S.d_ptype;
      bd.params = S.d_params;
    }
    CK(cudaEventRecord(S.h2d_done, db->h2d));
  }
  // kernels of this batch: after its upload, after the slot's previous outputs were read and
  // after the previous batch's compute (it may have run on another stream)
  CK(cudaStreamWaitEvent(s, S.out_ev, 0));
  if (db->submitted > 1) CK(cudaStreamWaitEvent(s, db->slots[(db->submitted - 2) % 3].comp_done, 0));
  if (timing) CK(cudaEventRecord(S.ev[0], s));
  // the slot's result words; the single-launch kernel writes them itself (word 0 too unless an
  // index catch-up below may raise an error in it first)
  const bool idx_catchup = db->idx_lag && (ops_mode || !db->olrow_ready);
  if (!small || idx_catchup) CK(cudaMemsetAsync(S.d_small, 0, 17 * sizeof(uint32_t), s));
  if (!n && !S.host_out) CK(cudaMemsetAsync(res->n_aborted, 0, sizeof(uint32_t), s));
  if (!b->inputs_on_device) CK(cudaStreamWaitEvent(s, S.h2d_done, 0));
  const bool packed_params = !ops_mode && b->proc_offsets;
  if (packed_params) bd.params = S.d_params;
  const size_t n_reads = ops_mode ? b->n_ops : (size_t)n * LTPG_PROC_RESULTS;
  const bool reads_dev = res->reads && res->outputs_on_device && !cr;
  long long* res_out = reads_dev ? reinterpret_cast<long long*>(res->reads) : S.d_res;
  uint32_t* counts = S.d_small + 8;
  // ---- work that depends on host-side state, stream-ordered ahead of the batch's device work ----
  // table metadata -> __constant__ (stream-ordered D2D; every TU holds its own copy);
  // skipped when this device's constant bank already holds this db's current tables
  if (g_uploaded[db->device % 64] != db->tab_version) {
    if (g_const_last[db->device % 64])  // the previous owner's kernels
      CK(cudaStreamWaitEvent(s, g_const_last[db->device % 64], 0));
    upload_tables_common(db->d_tab, s);
    upload_tables_ops(db->d_tab, s);
    upload_tables_tpcc(db->d_tab, s);
    g_uploaded[db->device % 64] = db->tab_version;
  }
  if ((db->cfg.flags & LTPG_FLAG_L2_PERSIST_MARKS) && db->persist_base) {
    // the largest mark array under a persisting L2 window (the set-aside is sized once from the
    // device's L2; accesses beyond the hit ratio stream)
    static size_t setaside = 0;
    if (!setaside) {
      int l2 = 0, maxw = 0;
      cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, db->device);
      cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxPersistingL2CacheSize, db->device);
      setaside = std::min<size_t>((size_t)maxw, std::min<size_t>(db->persist_bytes, (size_t)l2 / 2));
      if (setaside) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, setaside);
    }
    int maxwin = 0;
    cudaDeviceGetAttribute(&maxwin, cudaDevAttrMaxAccessPolicyWindowSize, db->device);
    cudaStreamAttrValue av{};
    av.accessPolicyWindow.base_ptr = db->persist_base;
    av.accessPolicyWindow.num_bytes = std::min<size_t>(db->persist_bytes, (size_t)maxwin);
    av.accessPolicyWindow.hitRatio =
        setaside ? std::min(1.0f, (float)setaside / (float)av.accessPolicyWindow.num_bytes) : 0.0f;
    av.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    av.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &av);
    cudaStreamSetAttribute(db->cap, cudaStreamAttributeAccessPolicyWindow, &av);
    cudaGetLastError();
  }
  if (db->epoch / 255 != db->mark_window) {  // the epoch tag byte wraps 0 -> 254: clear every mark
    db->mark_window = db->epoch / 255;
    for (uint32_t t = 0; t < db->n_tables; ++t) {
      const DevTable& T = db->h_tab[t];
      const size_t units = T.capacity * T.n_groups * sizeof(mark_t);
      if (T.wmarks) CK(cudaMemsetAsync(T.wmarks, 0xFF, units, s));
      if (T.rmarks) CK(cudaMemsetAsync(T.rmarks, 0xFF, units, s));
      if (T.amarks) CK(cudaMemsetAsync(T.amarks, 0xFF, T.capacity * __builtin_popcount(T.add_groups) * sizeof(mark_t), s));
      const uint64_t su_units[3] = {(uint64_t)T.sub_rows * T.n_groups,
                                    (uint64_t)T.sub_rows * __builtin_popcount(T.add_groups),
                                    (uint64_t)T.sub_rows * T.n_groups};
      for (int k = 0; k < 3; ++k)
        if (T.sub[k]) CK(cudaMemsetAsync(T.sub[k], 0xFF, su_units[k] * T.su * sizeof(mark_t), s));
    }
  }
  if (idx_catchup) {  // key lookups ahead: catch the indexes up
    for (uint32_t t = 0; t < db->n_tables; ++t)
      if ((db->idx_lag >> t) & 1u) launch_build_index_tail(t, db->d_idx_from + t, S.d_small, s);
    db->idx_lag = 0;
  }
  if (!ops_mode && !db->olrow_ready) {  // ORDER -> contiguous ORDER_LINE rows (first TPC-C batch)
    tpcc_build_olrow(s);
    db->olrow_ready = true;
  }
  if (!ops_mode && !((db->idx_lag >> LTPG_T_ORDER_LINE) & 1u) && db->h_tab[LTPG_T_ORDER_LINE].idx) {
    launch_note_rows(LTPG_T_ORDER_LINE, db->d_idx_from + LTPG_T_ORDER_LINE, s);  // first unindexed row
    db->idx_lag |= 1u << LTPG_T_ORDER_LINE;
  }
  const bool filter = !(db->cfg.flags & LTPG_FLAG_NO_MARK_FILTER);
  const bool reorder = (db->cfg.flags & LTPG_FLAG_REORDER) != 0;
  // fused OPS front end; NEXT-1 needs min reader marks on claimed keys, so it keeps the lists
  const bool fused = grouped && !reorder && !(db->cfg.flags & LTPG_FLAG_UNFUSED);
  std::vector<BatchDev> pb(L, bd);
  for (uint32_t p = 0; p < L; ++p) {
    Part& P = db->parts[p];
    BatchDev& x = pb[p];
    x.part = (uint32_t)db->cfg.rank * L + p;
    x.res = (!partitioned && p == 0) ? res_out : P.res;
    if (db->p2p && !sharded)  // own result slots live in the exchange region (peers pull them), by parity
      x.res = reinterpret_cast<long long*>(db->xregion + db->xl.off_res) + (uint64_t)(db->epoch & 1u) * db->xl.nres;
    if (sharded) x.res = res_out;  // every result slot is final on its home rank: written in place
    x.pmask = sharded ? P.pmask : nullptr;
    x.uref = P.uref;
    x.items = P.items;
    x.txn_ins = P.txn_ins;
    x.ua = P.ua;
    x.lflag = P.lflag;
    uint32_t* w = small ? small_words : P.small;
    x.err = w + 0;
    x.ins_tables = w + 1;
    x.kcount = w + 2;
    x.base = P.base;
    x.insdel = w + 12;
    x.done = w + 14;
  }
  S.h_vars->epoch = db->epoch;  // the slot's previous batch (the copy's last reader) is complete
  S.h_vars->clock = b->batch_clock;
  std::atomic_thread_fence(std::memory_order_seq_cst);
  // timing marks inside the batch's device work: event-record nodes when captured (always
  // recorded there, so one graph serves batches with and without statistics)
  bool capturing = false;
  auto tmark = [](cudaEvent_t e, cudaStream_t st) { return record_stage(e, st); };

  // ---- the batch's device work (a2..a8), enqueued on `s` -- or captured into a graph ---------
  auto enqueue = [&](cudaStream_t s) -> int {
    static_assert(MAXT <= 32, "k_batch_init clears the reservations with one warp");
    if (small) {
      if (tid_range) launch_fill_tid(S.d_tid + nc, nf, tid0, s);
      if (nc) {
        const Slot& P = db->slots[db->carry_slot];
        launch_carry(P.eff_tid, P.eff_ptype, P.eff_params, P.eff_abort, nc, S.d_tid, S.d_ptype, S.d_params, s);
        CK(cudaEventRecord(db->slots[db->carry_slot].comp_done, s));
      }
      BatchDev& x = pb[0];
      if (!ops_mode) {
        if (packed_params) {  // expand packed parameter blocks into 128-byte blocks (errors -> the slot's word)
          const uint8_t* packed = b->inputs_on_device ? b->proc_params : S.d_packed;
          const uint32_t* offs = b->inputs_on_device ? b->proc_offsets : S.d_offsets;
          uint8_t* dst = S.d_params + (size_t)nc * LTPG_PARAM_BYTES;
          if (b->flags & LTPG_BATCH_COMPACT_PARAMS) launch_unpack_compact(packed, offs, bd.ptype + nc, nf, dst, x.err, s);
          else launch_unpack_params(packed, offs, nf, dst, x.err, s);
        }
        // the batch scratch's rest state (a captured graph always carries the clears: it may be
        // replayed after a multi-kernel batch)
        if (!db->tpcc_small_clean || capturing) tpcc_small_clear(db->parts[0].tpcc, s);
      }
      const bool timed = timing || capturing;
      if (timed) CK(tmark(S.ev[1], s));
      x.status = st_out;
      if (ops_mode) {
        launch_ops_small(db->n_tables, x, filter, db->d_coop, db->d_reserve, S.d_vars,
                         capturing ? S.h_vars_dev : nullptr, db->epoch, b->batch_clock, bits_out, S.d_small,
                         !idx_catchup, abort_out, S.host_out ? nullptr : res->n_aborted, S.h_small_dev, small_bar, s);
      } else {
        const SmallOut so{db->d_reserve, S.d_vars, capturing ? S.h_vars_dev : nullptr, db->epoch, b->batch_clock,
                          bits_out, S.d_small, abort_out, S.host_out ? nullptr : res->n_aborted, S.h_small_dev,
                          !idx_catchup, small_bar};
        if (launch_tpcc_small(db->parts[0].tpcc, x, so, s)) return fail(db, LTPG_ECUDA, "k_tpcc_small launch failed");
      }
      if (timed)  // one kernel: ms_group holds the whole batch
        for (int e = 2; e <= 5; ++e) CK(tmark(S.ev[e], s));
      if (cr) launch_committed_reads(bits_out, n, res_out, cr_dst, db->d_wprefix, s);
      CK(cudaGetLastError());
      return LTPG_OK;
    }
    const uint32_t ib = std::min<uint32_t>(148u * 4u, std::max<uint32_t>(1u, (n / 16 + 255) / 256));
    k_batch_init<<<ib, 256, 0, s>>>(db->d_reserve, S.d_vars, capturing ? S.h_vars_dev : nullptr, db->epoch,
                                    b->batch_clock, db->parts[0].small, db->parts[0].ua, n,
                                    (ops_mode || !db->parts[0].tpcc.nw) ? nullptr : db->parts[0].tpcc.misc, db->parts[0].tpcc.dl_min,
                                    db->parts[0].tpcc.nw);
    note_launch();
    for (uint32_t p = 0; p < L; ++p) {
      Part& P = db->parts[p];
      if (p) {  // partition 0: cleared by k_batch_init
        CK(cudaMemsetAsync(P.small, 0, 16 * sizeof(uint32_t), s));
        if (n) CK(cudaMemsetAsync(P.ua, 0, n, s));
      }
      if (partitioned && n) {
        CK(cudaMemsetAsync(pb[p].res, 0, n_reads * sizeof(long long), s));
        CK(cudaMemsetAsync(P.lflag, 0, n, s));  // txns this partition does not touch: no verdict
      }
    }
    if (tid_range) launch_fill_tid(S.d_tid + nc, nf, tid0, s);  // consecutive TIDs of the given txns
    if (nc) {  // a9 on the device: the previous batch's conflict aborts lead this batch
      const Slot& P = db->slots[db->carry_slot];
      launch_carry(P.eff_tid, P.eff_ptype, P.eff_params, P.eff_abort, nc, S.d_tid, S.d_ptype, S.d_params, s);
      // the source slot's staging is reused only after this read (its next upload waits on it)
      CK(cudaEventRecord(db->slots[db->carry_slot].comp_done, s));
    }
    if (packed_params) {  // expand packed parameter blocks into 128-byte blocks (errors -> every partition)
      const uint8_t* packed = b->inputs_on_device ? b->proc_params : S.d_packed;
      const uint32_t* offs = b->inputs_on_device ? b->proc_offsets : S.d_offsets;
      uint8_t* dst = S.d_params + (size_t)nc * LTPG_PARAM_BYTES;
      if (b->flags & LTPG_BATCH_COMPACT_PARAMS)
        launch_unpack_compact(packed, offs, bd.ptype + nc, nf, dst, pb[0].err, s);
      else
        launch_unpack_params(packed, offs, nf, dst, pb[0].err, s);
      for (uint32_t p = 1; p < L; ++p) {
        k_copy_err<<<1, 1, 0, s>>>(pb[0].err, pb[p].err);
        note_launch();
      }
    }
    const bool timed = timing || capturing;
    if (timed) CK(tmark(S.ev[1], s));
    if (!n) return LTPG_OK;
    // ---- a1..a6 per partition: validate + warp division, claims, execute + marks, detect --------
    // NEXT-3 real-time popularity: OPS batches know T (every txn may access every table)
    // before their front end marks; TPC-C counts per procedure after grouping (tpcc_front)
    if (ops_mode) launch_popularity(db->h_tab, db->n_tables, nullptr, n, db->d_su, S.d_small + 11, s);
    for (uint32_t p = 0; p < L; ++p) {
      BatchDev& x = pb[p];
      cudaEvent_t* evp = (timed && p == L - 1) ? S.ev : nullptr;
      db->parts[p].tpcc.popular = S.d_small + 11;
      if (ops_mode) {
        if (fused) {  // validate + warp-local division + execute; INSERTs after their claims
          launch_ops_fused(db->n_tables, x, filter, s);
          if (evp) CK(tmark(evp[2], s));  // ms_group = the fused kernel; ms_exec = INSERT tail
          launch_ops_insert_tail(db->n_tables, x, filter, db->d_coop, s);  // one launch; no INSERT: returns
        } else {
          launch_ops_validate_group(db->n_tables, x, grouped, s);
          scan_exclusive_u32(x.txn_ins, x.txn_ins, n, db->d_scan, s, x.ins_tables);  // skipped: no INSERT
          launch_capacity_check(db->n_tables, x.ins_tables, x.txn_ins + n, x.base, x.reserve, x.err, s);
          launch_ops_claim(x, s);
          if (evp) CK(tmark(evp[2], s));
          launch_ops_exec(x, grouped, filter, s);
        }
        launch_bucket_reduce(db->h_tab, db->n_tables, db->d_su, s);  // NEXT-3 large-sized buckets (if any)
        if (evp) CK(tmark(evp[3], s));
        launch_ops_detect(x, s);
      } else {
        int rc = tpcc_front(db->parts[p].tpcc, x, s, evp, p == 0);  // partition 0: cleared by k_batch_init
        if (rc) return fail(db, rc, "tpcc launch failed");
      }
    }
    if (timed) CK(tmark(S.ev[4], s));
    // ---- exchange of per-txn verdicts (partitioned only) ---------------------------------------
    if (partitioned) {
      if (sharded) {  // bytes of cross-rank txns + remote-customer results, signal, wait + OR (xchg.cuh)
        launch_xput_sharded(pb[0].lflag, pb[0].pmask, bd.grank, bd.ptype, bd.params, pb[0].res, pb[0].err, n,
                            db->xpeers, db->xl, (uint32_t)db->cfg.rank, db->cfg.n_warehouses, db->epoch, db->d_xdone, s);
        launch_xcombine_sharded(db->xregion, db->xl, n, db->epoch, reorder, st_out, pb[0].lflag, pb[0].pmask,
                                bd.grank, bd.ptype, bd.params, pb[0].res, (uint32_t)db->cfg.rank, db->cfg.n_warehouses,
                                pb[0].err, S.d_small, s);
      } else if (db->p2p) {  // planes stored into every rank's region, signal, wait + OR (xchg.cuh)
        launch_xput(pb[0].lflag, pb[0].err, n, db->xpeers, db->xl, (uint32_t)db->cfg.rank, db->epoch, db->d_xdone, s);
        launch_xcombine(db->xregion, db->xl, n, db->epoch, reorder, st_out, pb[0].err, S.d_small, s);
      } else {  // loopback partitions of one process
        k_combine<<<(n + 255) / 256, 256, 0, s>>>(db->d_ptrs, L, n, st_out, db->d_ptrs + 64, S.d_small, reorder);
        k_spread_err<<<1, 1, 0, s>>>(S.d_small, db->d_ptrs + 64, L);
        note_launch(2);
      }
    }  // unpartitioned: the partition's error word reaches S.d_small with k_or_err after write-back
    if (timed) CK(tmark(S.ev[5], s));
    // ---- a8 on the finalize stream: commit bitmask, counts, abort list (status is final) ------
    CK(cudaEventRecord(db->status_ready, s));
    CK(cudaStreamWaitEvent(db->fin, db->status_ready, 0));
    launch_finalize_compact(st_out, n, bits_out, counts, S.d_small, abort_out, S.d_small + 16,
                            S.host_out ? nullptr : res->n_aborted, db->d_fc_state, db->d_fc_ctr, S.d_vars, db->fin);
    CK(cudaEventRecord(db->fin_done, db->fin));
    // ---- a7: write-back per partition -------------------------------------------------------
    for (uint32_t p = 0; p < L; ++p) {
      pb[p].status = st_out;
      if (ops_mode) {
        launch_ops_writeback(pb[p], db->n_tables, L == 1, s);  // L == 1: + the cursor advance
      } else {
        int rc = tpcc_back(db->parts[p].tpcc, pb[p], db->d_scan, s);
        if (rc) return fail(db, rc, "tpcc launch failed");
      }
    }
    if (ops_mode && L > 1)  // the combined verdict error, after every partition's write-back
      launch_advance_cursor(db->n_tables, db->d_reserve, S.d_small, db->d_dense_live, pb[0].insdel, s);
    // results: summed over partitions (each slot is written by its owning partition only)
    if (sharded) {
      // result slots final in place (home rank); nothing to sum
    } else if (db->p2p) {  // every rank publishes and reduces its slice (the protocol needs it)
      launch_xsig_res(db->xpeers, (uint32_t)db->cfg.rank, (uint32_t)db->cfg.world, db->epoch, s);
      launch_xsum(db->xpeers, db->xl, n_reads, db->epoch, res->reads ? res_out : db->d_xsink, S.d_small,
                  (uint32_t)db->cfg.rank, db->d_xdone + 1, s);
    } else if (partitioned && res->reads) {  // loopback partitions: sum of the partitions' slots
      k_sum_res<<<148 * 8, 256, 0, s>>>(db->d_ptrs + 128, L, n_reads, res_out);
      note_launch();
    }
    for (uint32_t p = 0; p < L && L > 1; ++p) {  // errors raised during write-back reach the caller
      k_or_err<<<1, 1, 0, s>>>(pb[p].err, S.d_small);  // too (one partition: k_publish ORs it in)
      note_launch();
    }
    CK(cudaStreamWaitEvent(s, db->fin_done, 0));
    if (cr) launch_committed_reads(bits_out, n, res_out, cr_dst, db->d_wprefix, s);  // bits and slots final
    CK(cudaGetLastError());
    return LTPG_OK;
  };

  // Graph replay: the same shape's captured graph if this slot has one, else capture, instantiate
  // and keep it (least recently used of GRAPHS_PER_SLOT replaced).  Multi-rank dbs enqueue
  // directly (their exchange selects buffers by epoch parity on the host).
  const bool use_graph = n && db->cfg.world == 1 && (db->cfg.flags & LTPG_FLAG_GRAPH) && !cr && !tid_range;
  if (use_graph) {
    GraphKey k;
    std::memset(&k, 0, sizeof(k));
    k.mode = b->mode, k.n = n, k.n_ops = bd.n_ops, k.bflags = b->flags & LTPG_BATCH_COMPACT_PARAMS;
    k.host_out = S.host_out, k.reads_dev = reads_dev, k.inputs_dev = b->inputs_on_device != 0;
    k.packed = packed_params;
    k.small_w0 = small && !idx_catchup;
    k.tab_version = db->tab_version;
    if (b->inputs_on_device) {
      const void* in[7] = {b->tid, b->op_begin, b->ops, b->op_arg, b->proc_type, b->proc_params, b->proc_offsets};
      std::memcpy(k.in, in, sizeof(in));
    }
    const void* outp[5] = {res->status, res->commit_bits, res->abort_idx, res->n_aborted, res->reads};
    if (!S.host_out) std::memcpy(k.out, outp, sizeof(outp));
    else k.out[4] = res->reads ? reinterpret_cast<const void*>(1) : nullptr;
    GraphEntry* E = nullptr;
    for (GraphEntry& g : S.graphs)
      if (g.exec && g.key == k) E = &g;
    if (!E) {  // capture on the private stream (the caller's may be the legacy default stream)
      E = &S.graphs[0];
      for (GraphEntry& g : S.graphs)
        if (!g.exec || g.last_use < E->last_use) E = &g;
      if (E->exec) {
        cudaGraphExecDestroy(E->exec);
        E->exec = nullptr;
      }
      const uint64_t l0 = g_kernel_launches;
      cudaGraph_t graph = nullptr;
      CK(cudaStreamBeginCapture(db->cap, cudaStreamCaptureModeThreadLocal));
      capturing = true;
      const int rc = enqueue(db->cap);
      capturing = false;
      const cudaError_t ec = cudaStreamEndCapture(db->cap, &graph);
      E->launches = g_kernel_launches - l0;
      g_kernel_launches = l0;
      if (rc) {
        if (graph) cudaGraphDestroy(graph);
        return rc;
      }
      if (ec != cudaSuccess) return fail(db, LTPG_ECUDA, std::string("graph capture: ") + cudaGetErrorString(ec));
      const cudaError_t ei = cudaGraphInstantiate(&E->exec, graph, 0);
      cudaGraphDestroy(graph);
      if (ei != cudaSuccess) {
        E->exec = nullptr;
        return fail(db, LTPG_ECUDA, std::string("cudaGraphInstantiate: ") + cudaGetErrorString(ei));
      }
      E->key = k;
    }
    E->last_use = ++db->graph_uses;
    CK(cudaGraphLaunch(E->exec, s));
    g_kernel_launches += E->launches;
  } else {
    const int rc = enqueue(s);
    if (rc) return rc;
  }
  if (!ops_mode && n) db->tpcc_small_clean = small;  // a multi-kernel batch leaves its scratch dirty
  if (timing) CK(cudaEventRecord(S.ev[6], s));
  CK(cudaEventRecord(S.comp_done, s));  // (also the next batch's "previous compute" and the constants' last user)
  g_const_last[db->device % 64] = S.comp_done;
  g_const_owner[db->device % 64] = db;
  // ---- a8: results: D2H on the copy stream (overlaps the next batch's kernels) ------------------
  cudaStream_t os = S.host_out ? db->d2h : s;
  if (S.host_out) CK(cudaStreamWaitEvent(db->d2h, S.comp_done, 0));
  const cudaMemcpyKind out_kind = S.host_out ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice;
  // error word, counters and abort count: one tiny kernel stores them into mapped host memory
  // (cheaper than a D2H copy in stream order); device outputs were written in place
  if (!small) {  // (the single-launch kernel's last block publishes them itself)
    k_publish<<<1, 32, 0, os>>>(S.d_small, S.h_small_dev, 17, L == 1 ? db->parts[0].small : nullptr);
    note_launch();
  }
  if (n && S.host_out) {
    if (res->status) CK(cudaMemcpyAsync(res->status, S.d_status, n, out_kind, os));
    CK(cudaMemcpyAsync(res->commit_bits, S.d_bits, ((n + 31) / 32) * sizeof(uint32_t), out_kind, os));
    if (res->reads && !reads_dev && !cr)
      CK(cudaMemcpyAsync(res->reads, res_out, n_reads * sizeof(int64_t), out_kind, os));
    if (res->abort_idx) CK(cudaMemcpyAsync(res->abort_idx, S.d_abort, n * sizeof(uint32_t), out_kind, os));
  } else if (n && res->reads && !reads_dev && !cr) {
    CK(cudaMemcpyAsync(res->reads, res_out, n_reads * sizeof(int64_t), out_kind, os));
  }
  // nothing after comp_done (single launch, device outputs, no statistics): it is the last event
  const bool tail = !small || S.host_out || timing || (n && res->reads && !reads_dev && !cr);
  S.out_ev = tail ? S.out_done : S.comp_done;
  if (tail) CK(cudaEventRecord(S.out_done, os));
  if (timing) res->stats->n_kernels = (uint32_t)(g_kernel_launches - S.launches0);
  S.eff_tid = bd.tid;
  S.eff_ptype = bd.ptype;
  S.eff_params = bd.params;
  S.eff_abort = abort_out;
  S.seq = db->submitted;
  S.carry_src = !ops_mode && db->cfg.world == 1 && db->loopback == 1;
  S.pending = true;
  if (async) return LTPG_OK;
  return finish_slot(db, S);
}

int ltpg_peer_handle(ltpg_db* db, void* out) {
  if (!db || !out) return LTPG_EINVAL;
  if (!db->p2p) return fail(db, LTPG_EINVAL, "no peer-memory exchange (world == 1)");
  CK(cudaSetDevice(db->device));
  PeerHandle h{};
  CK(cudaIpcGetMemHandle(&h.h, db->xregion));
  h.bytes = db->xl.bytes;
  h.magic = PEER_MAGIC;
  h.rank = (uint32_t)db->cfg.rank;
  h.world = (uint32_t)db->cfg.world;
  h.max_txns = db->cfg.max_txns;
  h.max_ops = db->cfg.max_ops;
  h.flags = db->cfg.flags;
  std::memcpy(out, &h, sizeof(h));
  return LTPG_OK;
}

int ltpg_connect_peers(ltpg_db* db, const void* handles) {
  if (!db || !handles) return LTPG_EINVAL;
  if (!db->p2p) return fail(db, LTPG_EINVAL, "no peer-memory exchange (world == 1)");
  if (db->connected) return fail(db, LTPG_EINVAL, "peers already connected");
  CK(cudaSetDevice(db->device));
  const uint32_t world = (uint32_t)db->cfg.world;
  std::vector<PeerHandle> hs(world);
  std::memcpy(hs.data(), handles, world * sizeof(PeerHandle));
  for (uint32_t q = 0; q < world; ++q) {
    const PeerHandle& h = hs[q];
    if (h.magic != PEER_MAGIC || h.rank != q || h.world != world || h.bytes != db->xl.bytes ||
        h.max_txns != db->cfg.max_txns || h.max_ops != db->cfg.max_ops || h.flags != db->cfg.flags)
      return fail(db, LTPG_EINVAL, "peer handle " + std::to_string(q) + " does not match this db's configuration");
  }
  for (uint32_t q = 0; q < world; ++q) {
    if (q == (uint32_t)db->cfg.rank) continue;
    void* p = nullptr;
    CK(cudaIpcOpenMemHandle(&p, hs[q].h, cudaIpcMemLazyEnablePeerAccess));
    db->opened.push_back(p);
    db->xpeers.base[q] = static_cast<char*>(p);
  }
  db->connected = true;
  return LTPG_OK;
}

int ltpg_mark_memory(ltpg_db* db, uint32_t t, uint64_t* standard_bytes, uint64_t* large_bytes, uint32_t* su) {
  if (!db || t >= db->n_tables || !standard_bytes || !large_bytes) return fail(db, LTPG_EINVAL, "bad mark_memory args");
  const DevTable& T = db->h_tab[t];
  const uint64_t na = __builtin_popcount(T.add_groups);
  *standard_bytes = (T.wmarks ? T.capacity * T.n_groups : 0) * sizeof(mark_t) +
                    (T.amarks ? T.capacity * na : 0) * sizeof(mark_t) +
                    (T.rmarks ? T.capacity * T.n_groups : 0) * sizeof(mark_t);
  const uint64_t units = (T.sub[0] ? (uint64_t)T.n_groups : 0) + (T.sub[1] ? na : 0) + (T.sub[2] ? (uint64_t)T.n_groups : 0);
  *large_bytes = T.su > 1 ? units * T.sub_rows * T.su * sizeof(mark_t) : 0;
  if (su) *su = T.su > 1 ? T.su : 1;
  return LTPG_OK;
}

int ltpg_dump_table(ltpg_db* db, uint32_t t, uint64_t* n_rows_out, uint64_t* keys, int64_t* cols) {
  if (!db || !n_rows_out || t >= db->n_tables) return fail(db, LTPG_EINVAL, "bad dump args");
  if (db->poisoned) return LTPG_EPOISONED;
  const DevTable& T = db->h_tab[t];
  if (!T.defined) return fail(db, LTPG_EINVAL, "table not loaded");
  CK(cudaSetDevice(db->device));
  CK(cudaDeviceSynchronize());
  unsigned long long nr = 0;
  CK(cudaMemcpy(&nr, T.n_rows, sizeof(nr), cudaMemcpyDeviceToHost));
  std::vector<uint8_t> valid(nr);
  if (nr) CK(cudaMemcpy(valid.data(), T.valid, nr, cudaMemcpyDeviceToHost));
  std::vector<uint64_t> rows;
  for (uint64_t r = 0; r < nr; ++r)
    if (valid[r]) rows.push_back(r);
  const uint64_t n = rows.size();
  if (!keys && !cols) {
    *n_rows_out = n;
    return LTPG_OK;
  }
  if (*n_rows_out < n) return fail(db, LTPG_EINVAL, "dump buffer too small");
  std::vector<unsigned long long> rk(T.has_pk ? nr : 0);
  if (T.has_pk && nr) CK(cudaMemcpy(rk.data(), T.rowkey, nr * 8, cudaMemcpyDeviceToHost));
  std::vector<std::vector<long long>> cv(T.n_cols, std::vector<long long>(nr));
  for (uint32_t c = 0; c < T.n_cols; ++c)
    if (nr) CK(cudaMemcpy2D(cv[c].data(), 8, T.col[c], 8ull * T.stride[c], 8, nr, cudaMemcpyDeviceToHost));
  if (T.has_pk) {
    std::sort(rows.begin(), rows.end(), [&](uint64_t a, uint64_t b) { return rk[a] < rk[b]; });
  } else {
    std::sort(rows.begin(), rows.end(), [&](uint64_t a, uint64_t b) {
      for (uint32_t c = 0; c < T.n_cols; ++c)
        if (cv[c][a] != cv[c][b]) return cv[c][a] < cv[c][b];
      return false;
    });
  }
  for (uint64_t i = 0; i < n; ++i) {
    if (T.has_pk && keys) keys[i] = rk[rows[i]];
    if (cols)
      for (uint32_t c = 0; c < T.n_cols; ++c) cols[c * n + i] = cv[c][rows[i]];
  }
  *n_rows_out = n;
  return LTPG_OK;
}

}  // extern "C"
