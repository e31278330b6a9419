// Internal device-side definitions of the B200 LTPG pipeline (not part of the ABI).
//
// HBM layout (DESIGN.md §"Data layout"):
//   * columns: int64, one array per column (SoA), `capacity` rows incl. the
//     append region; hidden `valid` byte and `rowkey` u64 per row;
//   * PK hash index: open addressing, linear probing, 16-byte slots
//     {u64 key, u32 row, u32 claim}, power-of-two size >= 2x capacity,
//     Fibonacci hashing (R6: the bucket function is result-invisible);
//   * conflict marks ("conflict log"): per (group,row) one 16-byte
//     record {u64 minW, u64 minA}; each u64 is epoch-tagged
//     ((0xFFFFFFFF - epoch) << 32 | rank) so a new batch never needs a reset
//     pass: u64 atomicMin keeps the newest epoch and, within it, the smallest
//     rank -- the per-unit minimum TID of P:219/P:225.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/ltpg.h"

namespace ltpg {

constexpr int MAXC = 16;
typedef uint32_t mark_t;
constexpr uint32_t MARK_RANK_BITS = 24;
constexpr int MAXT = 16;
constexpr uint64_t KEY_EMPTY = ~0ull;
constexpr uint32_t ROW_NONE = 0xFFFFFFFFu;
constexpr int NKINDS = 6;

// device error word bits
constexpr uint32_t ERR_EINVAL = 1u, ERR_ECAPACITY = 2u, ERR_EINTERNAL = 4u;

// check kinds stored in uref bits 62..63 (and bit 61 = "all groups")
constexpr uint64_t CHK_NONE = 0, CHK_RW = 1, CHK_A = 2, CHK_SCAN = 3;

struct alignas(16) IdxSlot {
  unsigned long long key;
  unsigned int row;
  unsigned int claim;
};

struct DevTable {
  long long* col[MAXC];
  uint32_t stride[MAXC];          // in int64 elements between consecutive rows
  uint8_t group[MAXC];
  uint8_t is_add[MAXC];
  uint32_t n_cols, n_groups;
  uint32_t has_pk, has_static, defined, owner_rule;
  uint64_t capacity;
  uint8_t* valid;
  unsigned long long* rowkey;
  // conflict marks, 32-bit epoch-tagged (mark_t): minW of every group, minA of the ADD
  // groups only (a plain group never receives an add), minR under NEXT-1 only
  mark_t* wmarks;                 // [n_groups][capacity]
  mark_t* amarks;                 // [popcount(add_groups)][capacity] or null
  mark_t* rmarks;                 // [n_groups][capacity] (LTPG_FLAG_REORDER only, else null)
  uint32_t add_groups;            // bit g: group g holds ADD columns
  IdxSlot* idx;
  uint64_t idx_mask;
  uint32_t idx_shift;
  unsigned long long* n_rows;     // device append cursor
  // warp-uniform forms of the per-column metadata (OPS path indexes columns by a
  // per-lane col id; dynamically indexed __constant__ arrays would serialise)
  // Row-block layout: each row has a "mutable" block of dstride words holding
  // its non-static columns in column order and a "static" block of sstride words holding
  // the static ones (blocks of <= 8 words padded to 1/2/4/8): the columns a procedure reads
  // or writes together share one sector / line.  The marks stay in their
  // own dense array: a mark RMW and the row's data read then miss on different lines and
  // are filled in parallel (measured: co-locating them serialises the two fills).
  long long* dyn;                 // [capacity][dstride]
  long long* stat;                // [capacity][sstride]
  uint32_t dstride, sstride;      // words per row block
  uint32_t dyn_mask;              // bit c: column c is non-static (lives in the mutable block)
  uint32_t columnar;              // LTPG_LAYOUT_COLUMNAR: column c at dyn + c * capacity
  uint64_t group_bits;            // 4 bits per column: group id, 15 = static
  uint32_t add_bits;              // bit c: column c is a delayed-ADD column
  // Dense key range (detected at load): key k in [key_base, key_base + dense_n) sits at row
  // k - key_base.  While the table has never seen an INSERT/DELETE (bit in *dense_live) a
  // lookup there is pure arithmetic -- the identity bucket function h(key) = key mod s_h
  // of P:217 on a dense key range -- and skips the hash-slot access.  Result-invisible (R6).
  uint64_t key_base, dense_n;
  uint32_t* aux;                  // TPC-C ORDER: first ORDER_LINE row of the order (ROW_NONE: probe)
  // NEXT-3 large-sized hash buckets (LTPG_FLAG_LARGE_BUCKETS): a popular table
  // (E = T/D > 1) records each mark in sub-slot (rank mod su) of its unit's bucket of su =
  // ceil(E/32)*32 sub-slots; k_bucket_reduce folds every bucket into the unit's mark word
  // before detection.  su <= 1: standard-sized (one slot per unit).
  // Popularity is identified per batch ("in real-time"): E = T/D with T = txns of the
  // batch that access the table, so a batch's bucket size c_su[id] = ceil(E/32)*32 (1: standard,
  // the mark word) is at most the allocated su (E bounded by max_txns / rows loaded).
  mark_t* sub[3];                 // [MK_W / MK_A / MK_R][group of that kind][sub_rows][su]
  uint32_t su;                    // allocated sub-slots per unit (the stride); <= 1: no buckets
  uint32_t sub_rows;              // rows with buckets (the rows loaded; appended rows: standard)
  uint32_t id;                    // table id (index of the batch's bucket size in c_su)
};

// table lookup honouring the dense mapping: dmask = *dense_live & ~(tables with INSERT/DELETE
// ops in this batch)
__device__ __forceinline__ bool lookup(const DevTable& T, uint32_t t, uint32_t dmask, uint64_t key, uint32_t& row,
                                       uint32_t& claim);

__device__ __forceinline__ uint32_t col_group(const DevTable& T, uint32_t c) {
  uint32_t g = (uint32_t)(T.group_bits >> (4 * c)) & 15u;
  return g == 15u ? LTPG_STATIC : g;
}
__device__ __forceinline__ bool col_is_add(const DevTable& T, uint32_t c) { return (T.add_bits >> c) & 1u; }
// column c of row, from per-table scalars only (OPS lanes index columns by a per-lane id)
__device__ __forceinline__ long long* col_ptr_ops(const DevTable& T, uint32_t c, uint32_t row) {
  if (T.columnar) return T.dyn + (uint64_t)c * T.capacity + row;
  const uint32_t below = (1u << c) - 1u;
  if ((T.dyn_mask >> c) & 1u)
    return T.dyn + (uint64_t)row * T.dstride + __popc(T.dyn_mask & below);
  return T.stat + (uint64_t)row * T.sstride + __popc(~T.dyn_mask & below);
}

__host__ __device__ inline uint64_t idx_hash(uint64_t key, uint32_t shift) {
  return (key * 0x9E3779B97F4A7C15ull) >> shift;
}

// Mark word = epoch tag (high 8 bits) | rank (low 24 bits; max_txns <= 2^24).  Batch e uses
// the tag byte 254 - (e mod 255): a later epoch has a smaller tag, so atomicMin overwrites
// older marks without a reset pass and mark_rank ignores them; the byte 0xFF (the
// "unmarked" value) never names a live epoch.  The byte wraps from 0 back to 254 every 255
// batches, so all marks are reset to 0xFF..FF before each such batch (capi.cu) -- 4 bytes per unit keep the
// mark arrays of the randomly touched tables L2-resident (126 MB) within a batch.
__host__ __device__ __forceinline__ uint32_t epoch_byte(uint32_t epoch) { return 254u - epoch % 255u; }
__device__ __forceinline__ mark_t epoch_tag(uint32_t epoch) { return epoch_byte(epoch) << MARK_RANK_BITS; }

// Minimum rank recorded for this epoch, or UINT32_MAX.
__device__ __forceinline__ uint32_t mark_rank(mark_t v, uint32_t epoch) {
  return (v >> MARK_RANK_BITS) == epoch_byte(epoch) ? (v & ((1u << MARK_RANK_BITS) - 1)) : 0xFFFFFFFFu;
}

// recordTID: atomicMin of this txn's rank into a mark word.  The
// plain pre-read skips the atomic when a smaller (or equal) rank is already
// there -- marks only decrease, so a stale read can only cause a redundant
// atomic, never a missing one (result-identical).
__device__ __forceinline__ void mark_min(mark_t* p, mark_t v, bool filter) {
  if (filter) {
    const mark_t cur = __ldcg(p);  // L2-coherent read, no system-scope fence
    if (cur <= v) return;
  }
  atomicMin(p, v);
}

__device__ __forceinline__ mark_t* wmark_ptr(const DevTable& T, uint32_t g, uint32_t row) {
  return T.wmarks + ((uint64_t)g * T.capacity + row);
}
// only for ADD groups (validated at load: ADD ops and ADD columns live in ADD groups)
__device__ __forceinline__ mark_t* amark_ptr(const DevTable& T, uint32_t g, uint32_t row) {
  return T.amarks + ((uint64_t)__popc(T.add_groups & ((1u << g) - 1u)) * T.capacity + row);
}
__device__ __forceinline__ mark_t* rmark_ptr(const DevTable& T, uint32_t g, uint32_t row) {
  return T.rmarks + ((uint64_t)g * T.capacity + row);
}

// recordTID into a unit's mark of kind k (write / add / read).  Standard-sized bucket: the
// mark word itself.  Large-sized bucket (NEXT-3): sub-slot h = TID mod s_u of the
// unit's bucket -- threads of different ranks mostly hit different words, so their atomics no
// longer serialise; k_bucket_reduce then takes the minimum over the bucket ("reads out
// all the TIDs in the hash bucket and selects ... the smallest TID").  Result-identical.
enum { MK_W = 0, MK_A = 1, MK_R = 2 };
static __constant__ uint16_t c_su[MAXT];  // this batch's bucket size per table (per TU copy)
__device__ __forceinline__ mark_t* mark_addr(const DevTable& T, int k, uint32_t g, uint32_t row, mark_t tag) {
  if (T.su > 1 && row < T.sub_rows) {
    const uint32_t su = c_su[T.id];
    if (su > 1) {
      const uint32_t gi = k == MK_A ? __popc(T.add_groups & ((1u << g) - 1u)) : g;
      return T.sub[k] + ((uint64_t)gi * T.sub_rows + row) * T.su + (tag & ((1u << MARK_RANK_BITS) - 1)) % su;
    }
  }
  return k == MK_W ? wmark_ptr(T, g, row) : (k == MK_A ? amark_ptr(T, g, row) : rmark_ptr(T, g, row));
}
__device__ __forceinline__ void mark_unit(const DevTable& T, int k, uint32_t g, uint32_t row, mark_t tag,
                                          bool filter) {
  mark_min(mark_addr(T, k, g, row, tag), tag, filter);
}

__device__ __forceinline__ long long* col_ptr(const DevTable& T, uint32_t c, uint32_t row) {
  return T.col[c] + (uint64_t)row * T.stride[c];
}

// Snapshot lookup: returns true if the key has a slot; row = ROW_NONE if absent
// in the snapshot (deleted / never inserted), claim = ROW_NONE unless an INSERT of
// this batch claimed it.
__device__ __forceinline__ bool idx_find(const DevTable& T, uint64_t key, uint32_t& row, uint32_t& claim) {
  uint64_t h = idx_hash(key, T.idx_shift);
  for (uint64_t probes = 0; probes <= T.idx_mask; ++probes) {
    const ulonglong2 v = *reinterpret_cast<const ulonglong2*>(T.idx + h);
    if (v.x == key) {
      row = (uint32_t)v.y;
      claim = (uint32_t)(v.y >> 32);
      return true;
    }
    if (v.x == KEY_EMPTY) break;
    h = (h + 1) & T.idx_mask;
  }
  row = ROW_NONE;
  claim = ROW_NONE;
  return false;
}

__device__ __forceinline__ bool lookup(const DevTable& T, uint32_t t, uint32_t dmask, uint64_t key, uint32_t& row,
                                       uint32_t& claim) {
  if (((dmask >> t) & 1u) && key - T.key_base < T.dense_n) {
    row = (uint32_t)(key - T.key_base);
    claim = ROW_NONE;
    return true;
  }
  return idx_find(T, key, row, claim);
}

// Find or create the slot of `key` (load / claim paths), probing from slot h.
__device__ __forceinline__ IdxSlot* idx_find_or_insert_from(const DevTable& T, uint64_t key, uint64_t h,
                                                            uint64_t probes0 = 0) {
  for (uint64_t probes = probes0; probes <= T.idx_mask; ++probes) {
    IdxSlot* s = T.idx + h;
    unsigned long long k = __ldcg(&s->key);  // hint only; the CAS decides
    if (k == KEY_EMPTY) k = atomicCAS(&s->key, KEY_EMPTY, key);
    if (k == KEY_EMPTY || k == key) return s;
    h = (h + 1) & T.idx_mask;
  }
  return nullptr;
}
__device__ __forceinline__ IdxSlot* idx_find_or_insert(const DevTable& T, uint64_t key) {
  return idx_find_or_insert_from(T, key, idx_hash(key, T.idx_shift));
}
// Two fresh keys in two tables (a NewOrder's ORDER and NEW_ORDER rows): both home slots are
// claimed by CAS straight away -- independent atomics, one round trip instead of a hint read
// and a CAS per key, one key after the other -- and only a taken home slot falls back to probing.
__device__ __forceinline__ void idx_insert2(const DevTable& TA, uint64_t ka, IdxSlot*& sa, const DevTable& TB,
                                            uint64_t kb, IdxSlot*& sb) {
  const uint64_t ha = idx_hash(ka, TA.idx_shift), hb = idx_hash(kb, TB.idx_shift);
  sa = TA.idx + ha;
  sb = TB.idx + hb;
  const unsigned long long va = atomicCAS(&sa->key, KEY_EMPTY, ka);
  const unsigned long long vb = atomicCAS(&sb->key, KEY_EMPTY, kb);
  if (va != KEY_EMPTY && va != ka) sa = idx_find_or_insert_from(TA, ka, (ha + 1) & TA.idx_mask, 1);
  if (vb != KEY_EMPTY && vb != kb) sb = idx_find_or_insert_from(TB, kb, (hb + 1) & TB.idx_mask, 1);
}

__device__ __forceinline__ IdxSlot* idx_slot(const DevTable& T, uint64_t key) {
  uint64_t h = idx_hash(key, T.idx_shift);
  for (uint64_t probes = 0; probes <= T.idx_mask; ++probes) {
    IdxSlot* s = T.idx + h;
    unsigned long long k = s->key;
    if (k == key) return s;
    if (k == KEY_EMPTY) return nullptr;
    h = (h + 1) & T.idx_mask;
  }
  return nullptr;
}

// uref: per-op record written by execute, read by detect / write-back.
//   bits  0..31 row (or claim row)   bits 32..39 group   bits 40..47 table
//   bit   59 write (CHK_RW: plain write; else a read)     bit 60 present in snapshot
//   bit   61 all groups              bits 62..63 check kind
__host__ __device__ __forceinline__ uint64_t make_uref(uint64_t chk, bool all, bool present, uint32_t t,
                                                       uint32_t g, uint32_t row, bool write = false) {
  return (chk << 62) | ((uint64_t)all << 61) | ((uint64_t)present << 60) | ((uint64_t)write << 59) |
         ((uint64_t)t << 40) | ((uint64_t)g << 32) | row;
}

// per-txn conflict bits (detect) and the verdict (R1; NEXT-1 reordering)
constexpr uint32_t CF_UA = 1u, CF_WAW = 2u, CF_RAW = 4u, CF_WAR = 8u;
enum { ACC_READ = 0, ACC_WRITE = 1, ACC_ADD = 2 };
__device__ __forceinline__ bool conflict_of(uint32_t bits, bool reorder) {
  return (bits & CF_WAW) || (reorder ? ((bits & CF_RAW) && (bits & CF_WAR)) : (bits & CF_RAW) != 0);
}
__device__ __forceinline__ uint8_t status_of_bits(uint32_t bits, bool reorder) {
  return conflict_of(bits, reorder) ? LTPG_ST_CONFLICT : ((bits & CF_UA) ? LTPG_ST_USER_ABORT : LTPG_ST_COMMIT);
}

// Conflict bits of one access of rank r to unit (g,row) (rcheck / wcheck; R1, R7):
//   READ  -> RAW if a smaller rank wrote or added
//   WRITE -> WAW if a smaller rank wrote or added; WAR if a smaller rank read (reorder only)
//   ADD   -> WAW if a smaller rank plainly wrote;  WAR if a smaller rank read (reorder only)
// The same on raw mark words: lim = epoch_tag(epoch) | r.  Within a mark window (capi.cu resets
// every mark when epoch / 255 changes) a live mark's tag byte is this epoch's or an older epoch's,
// i.e. >= this epoch's byte, so  mark_rank(v, epoch) < r  <=>  v < lim  (an older epoch's mark and
// the unmarked 0xFFFFFFFF compare above lim; r < 2^24) -- one compare per mark, no tag extraction.
__device__ __forceinline__ uint32_t unit_bits_lim(const DevTable& T, uint32_t g, uint32_t row, uint32_t acc,
                                                  mark_t lim) {
  const mark_t w = *wmark_ptr(T, g, row);
  const mark_t a = ((T.add_groups >> g) & 1u) ? *amark_ptr(T, g, row) : 0xFFFFFFFFu;
  const mark_t wa = w < a ? w : a;
  uint32_t bits = 0;
  if (acc == ACC_READ) return wa < lim ? CF_RAW : 0u;
  if ((acc == ACC_WRITE ? wa : w) < lim) bits |= CF_WAW;
  if (T.rmarks && *rmark_ptr(T, g, row) < lim) bits |= CF_WAR;
  return bits;
}
__device__ __forceinline__ uint32_t unit_bits(const DevTable& T, uint32_t g, uint32_t row, uint32_t acc, uint32_t r,
                                              uint32_t epoch) {
  return unit_bits_lim(T, g, row, acc, epoch_tag(epoch) | r);
}
__device__ __forceinline__ bool unit_conflicts(const DevTable& T, uint32_t g, uint32_t row, uint64_t chk,
                                               uint32_t r, uint32_t epoch) {
  return unit_bits(T, g, row, chk == CHK_A ? ACC_ADD : ACC_WRITE, r, epoch) & CF_WAW;
}

// Table metadata lives in __constant__ memory: warp-uniform table ids broadcast from
// the constant cache and are never evicted by the random data traffic (an ncu run
// showed per-op DevTable loads through L1 missing to L2).  Every translation unit
// has its own copy, uploaded stream-ordered before each batch (upload_tables_*).
static __constant__ DevTable c_tabs[MAXT];
#define LTPG_DEFINE_TABLE_UPLOAD(fn)                                                            \
  void fn(const DevTable* d, cudaStream_t s) { /* d: device copy -> async D2D */                \
    cudaMemcpyToSymbolAsync(c_tabs, d, sizeof(DevTable) * MAXT, 0, cudaMemcpyDeviceToDevice, s); \
  }                                                                                             \
  void fn##_su(const uint16_t* d_su, cudaStream_t s) { /* the batch's bucket sizes (NEXT-3) */   \
    cudaMemcpyToSymbolAsync(c_su, d_su, sizeof(uint16_t) * MAXT, 0, cudaMemcpyDeviceToDevice, s); \
  }
void upload_tables_common(const DevTable* h, cudaStream_t s);
void upload_tables_ops(const DevTable* h, cudaStream_t s);
void upload_tables_tpcc(const DevTable* h, cudaStream_t s);
void upload_tables_ops_su(const uint16_t* d_su, cudaStream_t s);
void upload_tables_tpcc_su(const uint16_t* d_su, cudaStream_t s);
void upload_tables_common_su(const uint16_t* d_su, cudaStream_t s);

// ---- host-side launchers (defined in the .cu files) ----------------------------------
// number of kernels launched by this library (reported per batch in ltpg_stats)
extern uint64_t g_kernel_launches;
inline void note_launch(uint32_t k = 1) { g_kernel_launches += k; }
// stage-timing event inside a batch's device work: an event-record node when the stream is
// being captured into a batch graph (a plain record there would only order the capture)
inline cudaError_t record_stage(cudaEvent_t e, cudaStream_t s) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaStreamIsCapturing(s, &cs);
  return cs == cudaStreamCaptureStatusActive ? cudaEventRecordWithFlags(e, s, cudaEventRecordExternal)
                                             : cudaEventRecord(e, s);
}

// Per-batch scalars that change from batch to batch while every pointer and size stays put.
// They live in device memory (one copy per pipeline slot, refreshed by a stream-ordered H2D
// copy of the slot's pinned host copy), so that a captured CUDA graph of the batch replays
// with the new values (capi.cu: graph replay).
struct BatchVars {
  uint32_t epoch, pad;
  long long clock;
};

struct BatchDev {
  // partitioning (§8(e)): nparts logical partitions (ranks x loopback); this is `part`.
  // nparts == 1: this partition owns everything and detect writes `status` directly;
  // otherwise detect writes lflag[r] = conflict bits (CF_*) for the exchange (OR over partitions).
  uint32_t nparts, part;
  uint32_t nw;                     // TPC-C: number of warehouses (warehouse ownership)
  uint64_t key_space;              // OPS: key-range ownership of owner_rule-2 tables
  uint8_t* lflag;                  // [n_txns] partitioned detect output
  unsigned long long* reserve;     // [MAXT] append rows reserved this batch (all partitions)
  unsigned long long* base;        // [MAXT] this partition's offset inside the reservation
  uint32_t* dense_live;            // persistent bitmask: tables whose dense mapping is valid
  uint32_t* insdel;                // this batch: tables receiving INSERT or DELETE ops (OPS)
  uint32_t* done;                  // zeroed per batch: block counter of the OPS write-back grid
  uint32_t n_txns, n_ops, flags;
  const BatchVars* vars;           // epoch (conflict-log tag) and batch clock, in device memory
  const unsigned long long* tid;
  const uint32_t* op_begin;
  const ltpg_op* ops;
  const long long* args;
  const uint8_t* ptype;
  const uint8_t* params;
  long long* res;            // OPS: [n_ops]   TPCC: [4 n]
  unsigned long long* uref;  // OPS: [n_ops]
  unsigned long long* items; // [NKINDS][max_ops]  (op idx | txn << 32)
  uint32_t* kcount;          // [NKINDS]
  uint32_t* txn_ins;         // [n_txns + 1] per-txn insert count -> exclusive offsets
  uint8_t* ua;               // [n_txns] user-abort flags
  uint8_t* status;           // [n_txns]
  uint32_t* err;             // device error word
  uint32_t* ins_tables;      // bitmask of tables receiving inserts
  uint32_t max_ops;
  // sharded TPC-C batches (include/ltpg.h): this rank's shard of a global batch.  Per-txn arrays
  // are indexed by the shard index i; the conflict TID (marks, checks) is the global rank
  // grank[i].  pmask[i]: the partitions txn i touches (k_tpcc_group, partitioned batches).
  const uint32_t* grank;           // null: the batch is the global batch (rank = index)
  uint32_t n_global;
  uint32_t* pmask;
};

// conflict TID of the batch's txn i (its global rank in a sharded batch)
__device__ __forceinline__ uint32_t grank_of(const BatchDev& b, uint32_t i) { return b.grank ? __ldg(b.grank + i) : i; }

__device__ __forceinline__ uint32_t b_epoch(const BatchDev& b) { return __ldg(&b.vars->epoch); }
__device__ __forceinline__ long long b_clock(const BatchDev& b) { return __ldg(&b.vars->clock); }

// "Last block" of a grid: every block calls this once at its end (after all of its threads'
// global writes); it returns true in exactly one block, the last to arrive, once every other
// block's writes are visible.  `ctr` is zeroed before the launch.
__device__ __forceinline__ bool last_block(uint32_t* ctr) {
  __shared__ bool last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd(ctr, 1u) == gridDim.x - 1;
    if (last) __threadfence();
  }
  __syncthreads();
  return last;
}

// ---- block-aggregated list reservation ------------------------------------------------------
// Every thread of a 256-thread block contributes cnt[k] items to list k; base[k] receives the
// global position of its first item.  One atomicAdd per block and list (per-warp atomics on
// a handful of counters serialised: ncu showed ~40% of a grouping kernel on them).
// FLAGS: bit k set = cnt[k] is 0 or 1 for every thread, so the warp scan is one ballot + popc
// instead of five shuffle steps.  Counters k < SPLIT live at counters0 + k, the others at
// counters1 + (k - SPLIT): one pair of block barriers for two counter arrays.
template <int NK, uint32_t FLAGS = 0u, int SPLIT = NK>
__device__ __forceinline__ void block_reserve(const uint32_t (&cnt)[NK], uint32_t* counters0, uint32_t (&base)[NK],
                                              uint32_t* counters1 = nullptr) {
  __shared__ uint32_t wsum[NK][8];
  __shared__ uint32_t gbase[NK];
  const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint32_t incl[NK];
#pragma unroll
  for (int k = 0; k < NK; ++k) {
    uint32_t x = cnt[k], tot;
    if ((FLAGS >> k) & 1u) {
      const uint32_t bal = __ballot_sync(0xffffffffu, x != 0u);
      x = __popc(bal & (0xffffffffu >> (31 - lane)));
      tot = __popc(bal);
      if (lane == 0) wsum[k][wid] = tot;
    } else {
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (uint32_t)o) x += y;
      }
      if (lane == 31) wsum[k][wid] = x;
    }
    incl[k] = x;
  }
  __syncthreads();
  if (threadIdx.x < NK) {
    const int k = threadIdx.x;
    uint32_t run = 0;
    for (int w = 0; w < 8; ++w) {
      const uint32_t v = wsum[k][w];
      wsum[k][w] = run;
      run += v;
    }
    gbase[k] = run ? atomicAdd(k < SPLIT ? counters0 + k : counters1 + (k - SPLIT), run) : 0u;
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < NK; ++k) base[k] = gbase[k] + wsum[k][wid] + incl[k] - cnt[k];
}

// ECAPACITY before anything mutates (one thread).  The partition's inserts take provisional rows
// n_rows + base + [0, total); base is this partition's offset in the batch reservation.  (Table
// metadata: the calling translation unit's c_tabs.)
__device__ __forceinline__ void capacity_body(uint32_t n_tables, const uint32_t* ins_tables, const uint32_t* total,
                                              unsigned long long* base, unsigned long long* reserve, uint32_t* err) {
  const uint32_t m = *ins_tables;
  const uint64_t tot = *total;
  for (uint32_t t = 0; t < n_tables; ++t) {
    base[t] = reserve[t];
    if ((m >> t) & 1u) {
      const DevTable& T = c_tabs[t];
      reserve[t] += tot;
      if (*T.n_rows + reserve[t] > T.capacity || *T.n_rows + reserve[t] > 0xFFFFFFF0ull) atomicOr(err, ERR_ECAPACITY);
    }
  }
}

// ---- ownership (contiguous ranges) -------------------------------------------------------
__host__ __device__ __forceinline__ uint32_t part_of_w(uint32_t w, uint32_t nw, uint32_t np) {
  return np <= 1 || !nw ? 0u : (uint32_t)(((uint64_t)(w - 1) * np) / nw);
}
__host__ __device__ __forceinline__ uint32_t part_of_key(uint32_t owner_rule, uint64_t key, uint64_t ks, uint32_t np) {
  if (np <= 1 || owner_rule != 2 || !ks) return 0u;  // rule 0/1 tables: partition 0 (OPS mode)
  const uint64_t chunk = (ks + np - 1) / np;
  const uint64_t p = key / chunk;
  return p >= np ? np - 1 : (uint32_t)p;
}
__device__ __forceinline__ bool owns_key(const BatchDev& b, const DevTable& T, uint64_t key) {
  return b.nparts <= 1 || part_of_key(T.owner_rule, key, b.key_space, b.nparts) == b.part;
}
__device__ __forceinline__ bool owns_w(const BatchDev& b, uint32_t w) {
  return b.nparts <= 1 || part_of_w(w, b.nw, b.nparts) == b.part;
}


// skip_if_zero (in-place scans only): when *skip_if_zero == 0 every input is 0, only out[n] = 0 is written
void scan_exclusive_u32(const uint32_t* in, uint32_t* out, uint32_t n, uint32_t* scratch, cudaStream_t s,
                        const uint32_t* skip_if_zero = nullptr);
void scan_exclusive_u64(const unsigned long long* in, unsigned long long* out, uint32_t n, uint32_t* scratch,
                        cudaStream_t s);
size_t scan_scratch_words(uint32_t n);

void launch_ops_validate_group(uint32_t n_tables, const BatchDev& b, bool grouped,
                               cudaStream_t s);
void launch_ops_claim(const BatchDev& b, cudaStream_t s);
void launch_ops_exec(const BatchDev& b, bool grouped, bool filter, cudaStream_t s);
void launch_ops_fused(uint32_t n_tables, const BatchDev& b, bool filter, cudaStream_t s);
void launch_ops_exec_inserts(const BatchDev& b, bool filter, cudaStream_t s);
// scan + capacity + claim + INSERT execution of the fused front end, one cooperative launch
uint32_t ops_small_max_txns();
void launch_ops_small(uint32_t n_tables, const BatchDev& b, bool filter, uint32_t* partials,
                      unsigned long long* reserve, BatchVars* vars, const volatile BatchVars* host, uint32_t epoch,
                      long long clock, uint32_t* commit_bits, uint32_t* dsmall, bool write0, uint32_t* abort_out,
                      uint32_t* n_out2, volatile uint32_t* host_small, uint32_t* bar, cudaStream_t s);
void launch_ops_insert_tail(uint32_t n_tables, const BatchDev& b, bool filter, uint32_t* partials, cudaStream_t s);
void launch_ops_detect(const BatchDev& b, cudaStream_t s);
void launch_ops_writeback(const BatchDev& b, uint32_t n_tables, bool advance, cudaStream_t s);
void launch_capacity_check(uint32_t n_tables, const uint32_t* ins_tables, const uint32_t* total,
                           unsigned long long* base, unsigned long long* reserve, uint32_t* err, cudaStream_t s);
void launch_advance_cursor(uint32_t n_tables, const unsigned long long* reserve, const uint32_t* err,
                           uint32_t* dense_live, const uint32_t* insdel, cudaStream_t s);
void launch_unpack_params(const uint8_t* packed, const uint32_t* offs, uint32_t n, uint8_t* params, uint32_t* err,
                          cudaStream_t s);
void launch_finalize(const uint8_t* status, uint32_t n, uint32_t* commit_bits, uint32_t* flags,
                     uint32_t* counts, const uint32_t* err, cudaStream_t s);
void launch_compact(const uint32_t* flags, const uint32_t* offs, uint32_t n, uint32_t* out, uint32_t* n_out,
                    uint32_t* n_out2, cudaStream_t s);
void launch_scatter_col(long long* dst, uint32_t stride, const long long* src, uint64_t n, cudaStream_t s);
void launch_committed_reads(const uint32_t* bits, uint32_t n, const long long* res, long long* out, uint32_t* pre,
                            cudaStream_t s);
void launch_fill_tid(unsigned long long* tid, uint32_t n, unsigned long long t0, cudaStream_t s);
void launch_carry(const unsigned long long* ptid, const uint8_t* ptype, const uint8_t* pparams, const uint32_t* abort,
                  uint32_t nc, unsigned long long* tid, uint8_t* type, uint8_t* params, cudaStream_t s);
void launch_unpack_compact(const uint8_t* packed, const uint32_t* offs, const uint8_t* types, uint32_t n,
                           uint8_t* params, uint32_t* err, cudaStream_t s);
// a8 in one kernel: commit bitmask, counts, abort list (decoupled look-back over 1024-txn tiles;
// tile_state[ceil(n/1024)] persists across batches, tile_ctr is reset on `s`)
void launch_finalize_compact(const uint8_t* status, uint32_t n, uint32_t* commit_bits, uint32_t* counts,
                             const uint32_t* err, uint32_t* out, uint32_t* n_out, uint32_t* n_out2,
                             unsigned long long* tile_state, uint32_t* tile_ctr, const BatchVars* vars, cudaStream_t s);
// NEXT-3: fold the large-sized buckets of every popular table into their units' mark words
// (host copies of the tables; nothing is launched when no table has su > 1)
void launch_bucket_reduce(const DevTable* h_tab, uint32_t n_tables, const uint16_t* d_su, cudaStream_t s);
// NEXT-3 real-time popularity: the batch's bucket size per table from T = txns accessing
// it and D = its loaded rows: su = E > 1 ? ceil(E/32)*32 : 1 with E = T/D, capped by the
// allocation; then copied into every TU's c_su; *popular = bitmask of tables with su > 1.
// kcount: TPC-C per-procedure list lengths (device) or null (OPS: T = n_all for every table).
// Nothing runs when no table has buckets.
void launch_popularity(const DevTable* h_tab, uint32_t n_tables, const uint32_t* kcount, uint32_t n_all,
                       uint16_t* d_su, uint32_t* popular, cudaStream_t s);
void launch_build_index_tail(uint32_t t, const unsigned long long* from, uint32_t* err, cudaStream_t s);
void launch_note_rows(uint32_t t, unsigned long long* dst, cudaStream_t s);
void launch_build_index(uint32_t t, uint64_t row0, uint64_t n, uint32_t* err,
                        cudaStream_t s);

}  // namespace ltpg
