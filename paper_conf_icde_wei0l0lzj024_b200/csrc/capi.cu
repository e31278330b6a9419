// C-ABI implementation (include/ltpg.h): device store management and the
// per-batch driver.  One ltpg_run_batch enqueues, on the caller's stream:
//   upload -> K-group -> [scan] -> K-claim -> K-exec -> K-detect -> [exchange]
//   -> K-wb -> finalize (commit bits, abort list) -> download
// The paper separates its three kernels with cudaDeviceSynchronize() (P:122,
// P:137-141); here stream order gives the same global isolation with no host
// round-trip inside the batch.
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <numeric>
#include <string>
#include <vector>

#include "ltpg_internal.cuh"
#include "tpcc_internal.cuh"

using namespace ltpg;

struct ltpg_db {
  ltpg_config cfg{};
  int device = 0;
  bool poisoned = false;
  std::string last_error;
  uint32_t epoch = 0;
  uint32_t n_tables = 0;
  uint64_t tab_version = 0;
  DevTable h_tab[MAXT]{};
  DevTable* d_tab = nullptr;
  unsigned long long* d_nrows = nullptr;  // [MAXT]
  // per-batch buffers
  unsigned long long* d_tid = nullptr;
  uint32_t* d_op_begin = nullptr;
  ltpg_op* d_ops = nullptr;
  long long* d_args = nullptr;
  uint8_t* d_ptype = nullptr;
  uint8_t* d_params = nullptr;
  long long* d_res = nullptr;
  unsigned long long* d_uref = nullptr;
  unsigned long long* d_items = nullptr;
  uint32_t* d_txn_ins = nullptr;
  uint8_t* d_ua = nullptr;
  uint8_t* d_status = nullptr;
  uint32_t* d_bits = nullptr;
  uint32_t* d_flags = nullptr;
  uint32_t* d_offs = nullptr;
  uint32_t* d_abort = nullptr;
  uint32_t* d_small = nullptr;  // [0]=err [1]=ins_tables [2..7] kcount [8..10] counts
  uint32_t* d_scan = nullptr;
  uint32_t* h_small = nullptr;  // pinned mirror of d_small (+ n_aborted)
  TpccDev tpcc{};
  cudaEvent_t ev[8]{};
};

namespace {

uint64_t g_tab_versions = 0;     // process-wide: every table load gets a new version
uint64_t g_uploaded[64] = {0};   // per device: version whose tables sit in __constant__

int fail(ltpg_db* db, int code, const std::string& msg) {
  if (db) {
    db->last_error = msg;
    if (code == LTPG_ECUDA || code == LTPG_ENCCL || code == LTPG_EINTERNAL) db->poisoned = true;
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
  if (T.col[0]) cudaFree(T.col[0]);
  if (T.valid) cudaFree(T.valid);
  if (T.rowkey) cudaFree(T.rowkey);
  if (T.marks) cudaFree(T.marks);
  if (T.idx) cudaFree(T.idx);
  unsigned long long* nr = T.n_rows;
  T = DevTable{};
  T.n_rows = nr;
}

}  // namespace

extern "C" {

const char* ltpg_version(void) { return "ltpg-b200 0.1 sm_100a"; }

const char* ltpg_last_error(const ltpg_db* db) { return db ? db->last_error.c_str() : "null db"; }

int ltpg_create_db(const ltpg_config* cfg, ltpg_db** out) {
  ltpg_db* db = nullptr;
  if (!cfg || !out) return LTPG_EINVAL;
  if (cfg->n_tables == 0 || cfg->n_tables > MAXT || cfg->max_txns == 0 || cfg->world < 1 ||
      cfg->rank < 0 || cfg->rank >= cfg->world || cfg->max_txns > (1u << 24) || cfg->max_ops > (1u << 24))
    return LTPG_EINVAL;
  db = new ltpg_db();
  db->cfg = *cfg;
  db->device = cfg->device;
  db->n_tables = cfg->n_tables;
  *out = db;
  CK(cudaSetDevice(cfg->device));
  const size_t n = cfg->max_txns, m = std::max<uint32_t>(cfg->max_ops, 1);
  CK(dmalloc(&db->d_tab, MAXT));
  CK(dmalloc(&db->d_nrows, MAXT));
  CK(cudaMemset(db->d_nrows, 0, MAXT * sizeof(unsigned long long)));
  for (int t = 0; t < MAXT; ++t) db->h_tab[t].n_rows = db->d_nrows + t;
  CK(dmalloc(&db->d_tid, n));
  CK(dmalloc(&db->d_op_begin, n + 1));
  CK(dmalloc(&db->d_ops, m));
  CK(dmalloc(&db->d_args, m));
  CK(dmalloc(&db->d_ptype, n));
  CK(dmalloc(&db->d_params, n * LTPG_PARAM_BYTES));
  CK(dmalloc(&db->d_res, std::max(m, n * LTPG_PROC_RESULTS)));
  CK(dmalloc(&db->d_uref, m));
  CK(dmalloc(&db->d_items, m * NKINDS));
  CK(dmalloc(&db->d_txn_ins, n + 1));
  CK(dmalloc(&db->d_ua, n));
  CK(dmalloc(&db->d_status, n));
  CK(dmalloc(&db->d_bits, (n + 31) / 32 + 1));
  CK(dmalloc(&db->d_flags, n));
  CK(dmalloc(&db->d_offs, n + 1));
  CK(dmalloc(&db->d_abort, n));
  CK(dmalloc(&db->d_small, 64));
  CK(dmalloc(&db->d_scan, scan_scratch_words(std::max<size_t>(n, m)) + 16));
  CK(cudaMallocHost(reinterpret_cast<void**>(&db->h_small), 64 * sizeof(uint32_t)));
  for (auto& e : db->ev) CK(cudaEventCreate(&e));
  CK(cudaMemcpy(db->d_tab, db->h_tab, sizeof(db->h_tab), cudaMemcpyHostToDevice));
  int rc = tpcc_alloc(db->tpcc, cfg->max_txns, cfg->n_warehouses);
  if (rc) return fail(db, rc, "tpcc scratch allocation failed (n_warehouses <= 1000)");
  return LTPG_OK;
}

void ltpg_destroy_db(ltpg_db* db) {
  if (!db) return;
  cudaSetDevice(db->device);
  cudaDeviceSynchronize();
  for (int t = 0; t < MAXT; ++t) free_table(db->h_tab[t]);
  void* bufs[] = {db->d_tab, db->d_nrows, db->d_tid, db->d_op_begin, db->d_ops, db->d_args, db->d_ptype,
                  db->d_params, db->d_res, db->d_uref, db->d_items, db->d_txn_ins, db->d_ua, db->d_status,
                  db->d_bits, db->d_flags, db->d_offs, db->d_abort, db->d_small, db->d_scan};
  for (void* p : bufs)
    if (p) cudaFree(p);
  if (db->h_small) cudaFreeHost(db->h_small);
  for (auto& e : db->ev)
    if (e) cudaEventDestroy(e);
  tpcc_free(db->tpcc);
  delete db;
}

int ltpg_load_table(ltpg_db* db, uint32_t t, const ltpg_table_desc* d, uint64_t n_rows, const uint64_t* keys,
                    const int64_t* cols) {
  if (!db) return LTPG_EINVAL;
  if (db->poisoned) return LTPG_EPOISONED;
  if (!d || t >= db->n_tables || d->n_cols > MAXC || (d->n_cols && (!d->col_group || !d->col_is_add)) ||
      n_rows > d->capacity_rows || d->capacity_rows >= 0xFFFFFFF0ull || (n_rows && d->n_cols && !cols) ||
      (d->has_pk && n_rows && !keys) || d->n_groups > 15)
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
  free_table(T);
  const uint64_t cap = std::max<uint64_t>(d->capacity_rows, 1);
  T.n_cols = d->n_cols;
  T.n_groups = d->n_groups;
  T.has_pk = d->has_pk ? 1 : 0;
  T.has_static = has_static;
  T.defined = 1;
  T.owner_rule = d->owner_rule;
  T.capacity = cap;
  long long* colmem = nullptr;
  CK(dmalloc(&colmem, cap * std::max<uint32_t>(d->n_cols, 1)));
  for (uint32_t c = 0; c < d->n_cols; ++c) {
    T.col[c] = colmem + c * cap;  // SoA: one contiguous int64 array per column
    T.stride[c] = 1;
    T.group[c] = d->col_group[c];
    T.is_add[c] = d->col_is_add[c] ? 1 : 0;
  }
  if (!d->n_cols) T.col[0] = colmem;
  T.col0 = colmem;
  T.group_bits = ~0ull;
  T.add_bits = 0;
  for (uint32_t c = 0; c < d->n_cols; ++c) {
    uint64_t g = d->col_group[c] == LTPG_STATIC ? 15u : d->col_group[c];
    T.group_bits = (T.group_bits & ~(15ull << (4 * c))) | (g << (4 * c));
    if (d->col_is_add[c]) T.add_bits |= 1u << c;
  }
  CK(dmalloc(&T.valid, cap));
  CK(cudaMemset(T.valid, 0, cap));
  CK(dmalloc(&T.rowkey, cap));
  if (d->n_groups) {
    CK(dmalloc(&T.marks, 2 * cap * d->n_groups));
    CK(cudaMemset(T.marks, 0xFF, 2 * cap * d->n_groups * sizeof(unsigned long long)));
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
    for (uint32_t c = 0; c < d->n_cols; ++c)
      CK(cudaMemcpy(T.col[c], cols + c * n_rows, n_rows * sizeof(int64_t), cudaMemcpyHostToDevice));
    CK(cudaMemset(T.valid, 1, n_rows));
    if (d->has_pk) CK(cudaMemcpy(T.rowkey, keys, n_rows * sizeof(uint64_t), cudaMemcpyHostToDevice));
  }
  unsigned long long nr = n_rows;
  CK(cudaMemcpy(T.n_rows, &nr, sizeof(nr), cudaMemcpyHostToDevice));
  CK(cudaMemcpy(db->d_tab, db->h_tab, sizeof(db->h_tab), cudaMemcpyHostToDevice));
  db->tab_version = ++g_tab_versions;
  if (d->has_pk && n_rows) {
    CK(cudaMemset(db->d_small, 0, sizeof(uint32_t)));
    upload_tables_common(db->d_tab, 0);
    g_uploaded[db->device % 64] = 0;
    launch_build_index(t, 0, n_rows, db->d_small, 0);
    CK(cudaGetLastError());
    uint32_t err = 0;
    CK(cudaMemcpy(&err, db->d_small, sizeof(err), cudaMemcpyDeviceToHost));
    if (err) {
      free_table(T);
      cudaMemcpy(db->d_tab, db->h_tab, sizeof(db->h_tab), cudaMemcpyHostToDevice);
      return fail(db, LTPG_EINVAL, "duplicate or reserved primary key");
    }
  }
  if (t == LTPG_T_CUSTOMER && db->cfg.n_warehouses) {
    int rc = tpcc_build_secondary(db->tpcc, keys, cols, n_rows, db->cfg.n_warehouses);
    if (rc) return fail(db, rc, "secondary index build failed");
  }
  CK(cudaDeviceSynchronize());
  return LTPG_OK;
}

int ltpg_run_batch(ltpg_db* db, const ltpg_batch* b, ltpg_result* res) {
  if (!db) return LTPG_EINVAL;
  if (db->poisoned) return LTPG_EPOISONED;
  if (!b || !res || !b->tid || !res->status || !res->commit_bits || !res->abort_idx || !res->n_aborted)
    return fail(db, LTPG_EINVAL, "null argument");
  const uint32_t n = b->n_txns;
  if (n > db->cfg.max_txns) return fail(db, LTPG_EINVAL, "n_txns > max_txns");
  const bool ops_mode = b->mode == LTPG_MODE_OPS;
  if (!ops_mode && b->mode != LTPG_MODE_TPCC) return fail(db, LTPG_EINVAL, "bad mode");
  if (ops_mode && (b->n_ops > db->cfg.max_ops || !b->op_begin || (b->n_ops && (!b->ops || !b->op_arg))))
    return fail(db, LTPG_EINVAL, "bad OPS batch");
  if (!ops_mode && (!b->proc_type || !b->proc_params || !db->cfg.n_warehouses))
    return fail(db, LTPG_EINVAL, "bad TPCC batch");
  CK(cudaSetDevice(db->device));
  cudaStream_t s = static_cast<cudaStream_t>(b->stream);
  const bool timing = res->stats != nullptr;
  if (timing) CK(cudaEventRecord(db->ev[0], s));
  ++db->epoch;
  const uint64_t launches0 = g_kernel_launches;
  BatchDev bd{};
  bd.n_txns = n;
  bd.n_ops = ops_mode ? b->n_ops : 0;
  bd.epoch = db->epoch;
  bd.flags = db->cfg.flags;
  bd.clock = b->batch_clock;
  bd.max_ops = std::max<uint32_t>(db->cfg.max_ops, 1);
  // ---- a1: upload -----------------------------------------------------------------
  const cudaMemcpyKind h2d = cudaMemcpyHostToDevice;
  if (b->inputs_on_device) {
    bd.tid = reinterpret_cast<const unsigned long long*>(b->tid);
    bd.op_begin = b->op_begin;
    bd.ops = b->ops;
    bd.args = reinterpret_cast<const long long*>(b->op_arg);
    bd.ptype = b->proc_type;
    bd.params = b->proc_params;
  } else {
    CK(cudaMemcpyAsync(db->d_tid, b->tid, n * sizeof(uint64_t), h2d, s));
    bd.tid = db->d_tid;
    if (ops_mode) {
      CK(cudaMemcpyAsync(db->d_op_begin, b->op_begin, (n + 1) * sizeof(uint32_t), h2d, s));
      if (b->n_ops) {
        CK(cudaMemcpyAsync(db->d_ops, b->ops, b->n_ops * sizeof(ltpg_op), h2d, s));
        CK(cudaMemcpyAsync(db->d_args, b->op_arg, b->n_ops * sizeof(int64_t), h2d, s));
      }
      bd.op_begin = db->d_op_begin;
      bd.ops = db->d_ops;
      bd.args = db->d_args;
    } else {
      CK(cudaMemcpyAsync(db->d_ptype, b->proc_type, n, h2d, s));
      CK(cudaMemcpyAsync(db->d_params, b->proc_params, (size_t)n * LTPG_PARAM_BYTES, h2d, s));
      bd.ptype = db->d_ptype;
      bd.params = db->d_params;
    }
  }
  const bool reads_dev = res->reads && res->outputs_on_device;
  bd.res = reads_dev ? reinterpret_cast<long long*>(res->reads) : db->d_res;
  bd.uref = db->d_uref;
  bd.items = db->d_items;
  bd.txn_ins = db->d_txn_ins;
  bd.ua = db->d_ua;
  bd.status = db->d_status;
  bd.err = db->d_small + 0;
  bd.ins_tables = db->d_small + 1;
  bd.kcount = db->d_small + 2;
  uint32_t* counts = db->d_small + 8;
  CK(cudaMemsetAsync(db->d_small, 0, 16 * sizeof(uint32_t), s));
  if (n) CK(cudaMemsetAsync(db->d_ua, 0, n, s));
  if (timing) CK(cudaEventRecord(db->ev[1], s));
  // table metadata -> __constant__ (stream-ordered D2D; every TU holds its own copy);
  // skipped when this device's constant bank already holds this db's current tables
  if (g_uploaded[db->device % 64] != db->tab_version) {
    upload_tables_common(db->d_tab, s);
    upload_tables_ops(db->d_tab, s);
    upload_tables_tpcc(db->d_tab, s);
    g_uploaded[db->device % 64] = db->tab_version;
  }
  const bool grouped = !(db->cfg.flags & LTPG_FLAG_NO_GROUPING);
  const bool filter = !(db->cfg.flags & LTPG_FLAG_NO_MARK_FILTER);
  if (n) {
    if (ops_mode) {
      // ---- a1/a2: validate + adaptive warp division ---------------------------------
      launch_ops_validate_group(db->n_tables, bd, grouped, s);
      scan_exclusive_u32(db->d_txn_ins, db->d_txn_ins, n, db->d_scan, s);
      launch_capacity_check(db->n_tables, bd.ins_tables, db->d_txn_ins + n, bd.err, s);
      // ---- a3: insert claims ----------------------------------------------------------
      launch_ops_claim(bd, s);
      if (timing) CK(cudaEventRecord(db->ev[2], s));
      // ---- a4/a5: execute + marks -----------------------------------------------------
      launch_ops_exec(bd, grouped, filter, s);
      if (timing) CK(cudaEventRecord(db->ev[3], s));
      // ---- a6: conflict detection -------------------------------------------------------
      launch_ops_detect(bd, s);
      if (timing) CK(cudaEventRecord(db->ev[4], s));
      if (timing) CK(cudaEventRecord(db->ev[5], s));
      // ---- a7: write-back -------------------------------------------------------------
      launch_ops_writeback(bd, s);
      launch_advance_cursor(db->n_tables, bd.ins_tables, db->d_txn_ins + n, bd.err, s);
    } else {
      int rc = tpcc_run(db->tpcc, bd, db->d_scan, s, timing ? db->ev : nullptr);
      if (rc) return fail(db, rc, "tpcc launch failed");
    }
    // ---- finalize: commit bitmask, abort list ------------------------------------------
    launch_finalize(db->d_status, n, db->d_bits, db->d_flags, counts, bd.err, s);
    scan_exclusive_u32(db->d_flags, db->d_offs, n, db->d_scan, s);
    launch_compact(db->d_flags, db->d_offs, n, db->d_abort, s);
  }
  CK(cudaGetLastError());
  if (timing) CK(cudaEventRecord(db->ev[6], s));
  // ---- a8: results --------------------------------------------------------------------
  const cudaMemcpyKind out_kind = res->outputs_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost;
  CK(cudaMemcpyAsync(db->h_small, db->d_small, 16 * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
  if (n) {
    CK(cudaMemcpyAsync(db->h_small + 16, db->d_offs + n, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(res->status, db->d_status, n, out_kind, s));
    CK(cudaMemcpyAsync(res->commit_bits, db->d_bits, ((n + 31) / 32) * sizeof(uint32_t), out_kind, s));
    if (res->reads && !reads_dev) {
      size_t nr = ops_mode ? b->n_ops : (size_t)n * LTPG_PROC_RESULTS;
      CK(cudaMemcpyAsync(res->reads, db->d_res, nr * sizeof(int64_t), out_kind, s));
    }
    if (res->outputs_on_device) {
      CK(cudaMemcpyAsync(res->n_aborted, db->d_offs + n, sizeof(uint32_t), out_kind, s));
      CK(cudaMemcpyAsync(res->abort_idx, db->d_abort, n * sizeof(uint32_t), out_kind, s));
    }
  } else {
    db->h_small[16] = 0;
  }
  CK(cudaStreamSynchronize(s));
  const uint32_t err = db->h_small[0];
  if (err & ERR_EINTERNAL) return fail(db, LTPG_EINTERNAL, "device invariant violated");
  if (err & ERR_EINVAL) return fail(db, LTPG_EINVAL, "invalid batch (validated on device; nothing changed)");
  if (err & ERR_ECAPACITY) return fail(db, LTPG_ECAPACITY, "append capacity exceeded (nothing changed)");
  const uint32_t n_ab = db->h_small[16];
  if (!res->outputs_on_device) {
    *res->n_aborted = n_ab;
    if (n_ab) CK(cudaMemcpyAsync(res->abort_idx, db->d_abort, n_ab * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
  }
  if (timing) {
    CK(cudaEventRecord(db->ev[7], s));
    CK(cudaEventSynchronize(db->ev[7]));
    ltpg_stats* st = res->stats;
    float ms[7] = {0};
    for (int i = 0; i < 7; ++i) CK(cudaEventElapsedTime(&ms[i], db->ev[i], db->ev[i + 1]));
    st->ms_upload = ms[0];
    st->ms_group = ms[1];
    st->ms_exec = ms[2];
    st->ms_detect = ms[3];
    st->ms_exchange = ms[4];
    st->ms_writeback = ms[5];
    st->ms_download = ms[6];
    st->n_commit = db->h_small[8];
    st->n_conflict = db->h_small[9];
    st->n_user_abort = db->h_small[10];
    st->n_kernels = (uint32_t)(g_kernel_launches - launches0);
  }
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
