// TPC-C PROC mode: pre-compiled stored procedures decomposed into typed
// sub-transactions and run by type-homogeneous warps (adaptive warp division,
// P:195-199, Fig. 3):
//   NewOrder    16 lanes / txn: lane l < n = order line l (item + stock RMW), lane 15 = header
//   Payment      1 lane  / txn
//   OrderStatus 16 lanes / txn: lane 15 = customer + order, lanes < cnt = order lines
//   Delivery    16 lanes / txn: lane d-1 = district d
//   StockLevel  32 lanes / txn: lanes over the 20-order window, then over distinct items
// Every procedure is one template instantiated for the three phases of Alg. 1:
//   PH_EXEC    readMem / recordLS / recordTID (marks)
//   PH_DETECT  rcheck / wcheck over the same units
//   PH_WB      writeMem of committed txns
// so the unit set checked is by construction the unit set marked.  Rows found by
// execute are logged (NewOrder / Payment / OrderStatus) and reused; Delivery and
// StockLevel re-derive their rows (their lookups are static or own-unit reads).
// NewOrder's fetch-ADD of D_NEXT_O_ID (R12, delayed-update prefix sum P:241) is
// resolved after detection by a per-district prefix count in rank order.
#include <algorithm>
#include <cstdio>
#include <map>
#include <vector>

#include "tpcc_internal.cuh"

namespace ltpg {

LTPG_DEFINE_TABLE_UPLOAD(upload_tables_tpcc)

enum { PH_EXEC = 0, PH_DETECT = 1, PH_WB = 2 };

#ifdef LTPG_SMALL_TS  // diagnostic builds: per-stage times, printed by the last block
__device__ unsigned long long g_tsm[2][10];  // [0][k]: block 0 passed barrier k; [1][k]: latest work end of stage k
#define TSM_PASS(k) \
  if (blockIdx.x == 0 && threadIdx.x == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g_tsm[0][k]))
#define TSM_AT(k)                                                \
  {                                                              \
    unsigned long long t_;                                       \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));       \
    atomicMax(&g_tsm[1][k], t_);                                 \
  }
#define TSM_WORK(k)                                              \
  {                                                              \
    __syncthreads();                                             \
    unsigned long long t_;                                       \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));       \
    if (threadIdx.x == 0) atomicMax(&g_tsm[1][k], t_);           \
  }
#else
#define TSM_PASS(k)
#define TSM_WORK(k)
#define TSM_AT(k)
#endif

__device__ __forceinline__ uint32_t p16(const uint8_t* p, int off) { return *reinterpret_cast<const uint16_t*>(p + off); }
__device__ __forceinline__ uint32_t p32(const uint8_t* p, int off) { return *reinterpret_cast<const uint32_t*>(p + off); }
__device__ __forceinline__ long long p64(const uint8_t* p, int off) { return *reinterpret_cast<const long long*>(p + off); }

__device__ __forceinline__ uint64_t kD(uint64_t w, uint64_t d) { return w * 10 + d; }
__device__ __forceinline__ uint64_t kC(uint64_t w, uint64_t d, uint64_t c) { return kD(w, d) * 3000 + c; }
__device__ __forceinline__ uint64_t kS(uint64_t w, uint64_t i) { return w * 100000 + i; }
__device__ __forceinline__ uint64_t kO(uint64_t w, uint64_t d, uint64_t o) { return (kD(w, d) << 32) | o; }

__device__ __forceinline__ uint32_t probe(const DevTable& T, uint64_t key) {
  uint32_t row, claim;
  idx_find(T, key, row, claim);
  return row;
}
// Two-step probe so independent lookups of one lane are in flight together (the exec
// kernel is bound by dependent index -> row -> column latency; ncu: ~32% of stall samples
// sat on the first slot load): issue the first slot loads, then resolve them.
__device__ __forceinline__ ulonglong2 probe_issue(const DevTable& T, uint64_t key, uint64_t& h) {
  h = idx_hash(key, T.idx_shift);
  return *reinterpret_cast<const ulonglong2*>(T.idx + h);
}
__device__ __forceinline__ uint32_t probe_finish(const DevTable& T, uint64_t key, uint64_t h, ulonglong2 v) {
  for (uint64_t probes = 0; probes <= T.idx_mask; ++probes) {
    if (v.x == key) return (uint32_t)v.y;
    if (v.x == KEY_EMPTY) return ROW_NONE;
    h = (h + 1) & T.idx_mask;
    v = *reinterpret_cast<const ulonglong2*>(T.idx + h);
  }
  return ROW_NONE;
}
// pending lookup honouring the dense key->row mapping of W/D/C/I/S (no slot access there)
struct PP {
  uint64_t key, h;
  ulonglong2 v;
  uint32_t row;
};
__device__ __forceinline__ PP pp_issue(const DevTable& T, uint32_t t, uint64_t key, uint32_t dmask) {
  PP p;
  p.key = key;
  if (((dmask >> t) & 1u) && key - T.key_base < T.dense_n) {
    p.row = (uint32_t)(key - T.key_base);
    p.h = ~0ull;
  } else {
    p.row = ROW_NONE;
    p.v = probe_issue(T, key, p.h);
  }
  return p;
}
__device__ __forceinline__ uint32_t pp_finish(const DevTable& T, const PP& p) {
  return p.h == ~0ull ? p.row : probe_finish(T, p.key, p.h, p.v);
}
__device__ __forceinline__ uint32_t rowof(const DevTable& T, uint32_t t, uint64_t key, uint32_t dmask) {
  uint32_t row, claim;
  lookup(T, t, dmask, key, row, claim);
  return row;
}
__device__ __forceinline__ long long rd(const DevTable& T, uint32_t c, uint32_t row) { return *col_ptr(T, c, row); }
__device__ __forceinline__ void wr(const DevTable& T, uint32_t c, uint32_t row, long long v) { *col_ptr(T, c, row) = v; }
// STOCK's four counters side by side in one 32-byte row block (row-block layout: S_QUANTITY,
// S_YTD, S_ORDER_CNT, S_REMOTE_CNT at consecutive words, 16-byte aligned rows)
__device__ __forceinline__ bool stock_block_vec(const DevTable& T) {
  return !T.columnar && T.stride[S_QUANTITY] == 4 && T.col[S_YTD] == T.col[S_QUANTITY] + 1 &&
         T.col[S_ORDER_CNT] == T.col[S_QUANTITY] + 2 && T.col[S_REMOTE_CNT] == T.col[S_QUANTITY] + 3 &&
         (reinterpret_cast<uintptr_t>(T.col[S_QUANTITY]) & 15u) == 0;
}
// write-back increment: an ADD-unit column may have several committed adders (atomic); a
// WRITE-unit column has exactly one committed writer per batch (R1: WAW) -> plain RMW
__device__ __forceinline__ void addv(const DevTable& T, uint32_t c, uint32_t row, long long v) {
  long long* p = col_ptr(T, c, row);
  if (col_is_add(T, c)) atomicAdd(reinterpret_cast<unsigned long long*>(p), (unsigned long long)v);
  else *p = (long long)((unsigned long long)*p + (unsigned long long)v);
}

struct Tx {
  uint32_t dmask;  // tables with a live dense key->row mapping
  uint32_t r;
  uint32_t epoch;
  mark_t tag;
  bool filter;
  uint32_t bits;   // detect: conflict bits found so far (CF_*)
  uint32_t* err;
  bool reorder;    // NEXT-1 logical reordering
  mark_t* hm;      // execute: the block's shared-memory marks of the WAREHOUSE / DISTRICT units (or null)
  uint32_t nw;
  // verdict already decided by the bits found (remaining checks cannot change it)
  __device__ __forceinline__ bool done() const { return conflict_of(bits, reorder); }
};

__device__ __forceinline__ void internal_error(Tx& x) { atomicOr(x.err, ERR_EINTERNAL); }

// unit actions per phase: plain write (W mark / RW check), delayed add (A mark / A check),
// marked read (RW check only; reads leave no mark under R1)
// Marks: the read-before-atomicMin filter is applied to the popular tables only (P:215,
// E = T/D > 1: WAREHOUSE and DISTRICT, thousands of accesses per row and batch); on cold
// rows it would add a dependent DRAM round trip before a fire-and-forget RED.
// Execute: the hottest units -- WAREHOUSE (W_YTD) and DISTRICT (D_YTD, D_NEXT_O_ID, the
// Delivery cursor), touched by nearly every txn -- are marked into a per-block shared-memory
// copy (atomicMin in shared memory, hm) and flushed with one global atomicMin per touched unit
// when the block ends (k_tpcc_phase): marks are read only by detection, after this kernel, and
// min is order-free, so the marks are identical; the per-txn filter read of a hot L2 line (a
// dependent round trip, ~11% of execute's stall samples) disappears.  A unit whose group kind
// does not match (a W mark on an ADD group) takes the global path.
__device__ __forceinline__ mark_t* hot_mark(const DevTable& T, uint32_t g, uint32_t row, const Tx& x, bool add) {
#ifdef LTPG_NO_HOT_MARKS
  return nullptr;
#endif
  if (!x.hm || T.id > TD || (((T.add_groups >> g) & 1u) != (add ? 1u : 0u))) return nullptr;
  if (T.id == TW) return (g == 0 && row < x.nw) ? x.hm + row : nullptr;
  return (g < 3 && row < 10 * x.nw) ? x.hm + x.nw + g * 10 * x.nw + row : nullptr;
}
template <int PH>
__device__ __forceinline__ void unit_w(const DevTable& T, uint32_t g, uint32_t row, Tx& x, bool hot = false) {
  if (PH == PH_EXEC) {
    mark_t* h = hot ? hot_mark(T, g, row, x, false) : nullptr;
    if (h) atomicMin(h, x.tag);
    else mark_unit(T, MK_W, g, row, x.tag, x.filter && hot);
  }
  if (PH == PH_DETECT && !x.done()) x.bits |= unit_bits_lim(T, g, row, ACC_WRITE, x.tag);
}
template <int PH>
__device__ __forceinline__ void unit_a(const DevTable& T, uint32_t g, uint32_t row, Tx& x, bool hot = false) {
  if (PH == PH_EXEC) {
    mark_t* h = hot ? hot_mark(T, g, row, x, true) : nullptr;
    if (h) atomicMin(h, x.tag);
    else mark_unit(T, MK_A, g, row, x.tag, x.filter && hot);
  }
  if (PH == PH_DETECT && !x.done()) x.bits |= unit_bits_lim(T, g, row, ACC_ADD, x.tag);
}
template <int PH>
__device__ __forceinline__ void unit_r(const DevTable& T, uint32_t g, uint32_t row, Tx& x, bool hot = false) {
  if (g == LTPG_STATIC) return;
  if (PH == PH_EXEC && T.rmarks) mark_unit(T, MK_R, g, row, x.tag, x.filter && hot);  // NEXT-1 minR
  if (PH == PH_DETECT && !x.done()) x.bits |= unit_bits_lim(T, g, row, ACC_READ, x.tag);
}
// update of column c (strict: WRITE unit of its group; delayed: ADD unit)
template <int PH>
__device__ __forceinline__ void col_upd(const DevTable& T, uint32_t c, uint32_t row, Tx& x, bool hot = false) {
  if (col_is_add(T, c)) unit_a<PH>(T, col_group(T, c), row, x, hot);
  else unit_w<PH>(T, col_group(T, c), row, x, hot);
}
// same for columns c1..c3 updated together; a unit shared by several columns is touched once
template <int PH>
__device__ __forceinline__ void col_upd3(const DevTable& T, uint32_t c1, uint32_t c2, uint32_t c3, uint32_t row,
                                         Tx& x, bool hot = false) {
  const uint32_t g1 = col_group(T, c1), g2 = col_group(T, c2), g3 = col_group(T, c3);
  col_upd<PH>(T, c1, row, x, hot);
  if (g2 != g1) col_upd<PH>(T, c2, row, x, hot);
  if (g3 != g1 && g3 != g2) col_upd<PH>(T, c3, row, x, hot);
}

__device__ __forceinline__ long long seg16_sum(long long v) {
#pragma unroll
  for (int o = 8; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o, 16);
  return v;
}
__device__ __forceinline__ uint32_t seg16_or(uint32_t v) {
#pragma unroll
  for (int o = 8; o; o >>= 1) v |= __shfl_xor_sync(0xffffffffu, v, o, 16);
  return v;
}

// ECAPACITY before write-back: worst case every NewOrder / Payment of this partition
// commits; partitions of one process share the table and reserve in stream order (one thread
// of the execute grid's first block, after the grouping kernel)
__device__ void tpcc_capacity_tail(const BatchDev& b, const TpccParams& tp) {
  const uint64_t add[4] = {__ldcg(tp.misc + M_NO), __ldcg(tp.misc + M_NO), __ldcg(tp.misc + M_NO_LINES),
                           __ldcg(tp.misc + M_PAY)};
  const int tabs[4] = {TO, TNO, TOL, TH};
  for (int k = 0; k < 4; ++k) {
    const DevTable& T = c_tabs[tabs[k]];
    b.reserve[tabs[k]] += add[k];
    if (*T.n_rows + b.reserve[tabs[k]] > T.capacity) atomicOr(b.err, ERR_ECAPACITY);
  }
}

// append-row counters advanced past this batch's committed rows (one thread of the write-back
// phase's last block)
__device__ void tpcc_advance_tail(const BatchDev& b, const TpccParams& tp) {
  if (*(volatile uint32_t*)b.err) return;
  const uint32_t n = b.n_txns;
  const unsigned long long tot = __ldcg(tp.no_pref + n);
  *c_tabs[TO].n_rows += (uint32_t)tot;
  *c_tabs[TNO].n_rows += (uint32_t)tot;
  *c_tabs[TOL].n_rows += tot >> 32;
  *c_tabs[TH].n_rows += __ldcg(tp.misc + M_HIST);
}

// chunk_cnt[chunk][district] word: district-major ([dk][chunk]) up to COLSCAN_TILED_DSZ district
// keys and on the single-launch path -- the column scan reads whole rows coalesced (chunk-major,
// a warp reading one word per 2.6 KB row: 16.5 us on tpcc_c4; tpcc_c2 single launch 9 -> 5 us;
// tpcc_c4 write-back 0.128 -> 0.124 ms, profiles/ab_r02_assign.txt) -- chunk-major above (512
// warehouses: the per-chunk histogram's 5131 scattered stores per chunk would cost more than the
// tiled column scan, k_no_colscan_tiled, that transposes through shared memory)
__device__ __forceinline__ uint64_t cc_at(const TpccParams& tp, uint32_t dk, uint32_t c) {
  return tp.cc_dm ? (uint64_t)dk * tp.n_chunks + c : (uint64_t)c * tp.dsz + dk;
}
// a committed NewOrder's o_id (the fetch-ADD pre-image of D_NEXT_O_ID, R12): assigned by k_no_assign
// into its first result slot, or -- single-launch path (oid_inline, 32-rank chunks) -- the
// district's snapshot value + committed NewOrders of the district in earlier chunks (column
// scan) + those of smaller rank in the txn's own chunk (dk_of, written by no_chunk32_body)
__device__ __forceinline__ long long no_oid(const BatchDev& b, const TpccParams& tp, uint32_t r, uint32_t w, uint32_t d) {
  if (!tp.oid_inline) return b.res[4ull * r];
  const uint32_t dk = (uint32_t)kD(w, d);
  return tp.dist_base[dk] + tp.chunk_cnt[cc_at(tp, dk, r >> tp.chunk_shift)] + tp.dk_of[r];
}

// ---- NewOrder (TPC-C 2.4; SURVEY §8(c) procedure table) --------------------------------
template <int PH>
__device__ void proc_neworder(const BatchDev& b, const TpccParams& tp, uint32_t r, uint32_t sub, bool active, Tx& x) {
  const DevTable& TWh = c_tabs[TW];
  const DevTable& TDi = c_tabs[TD];
  const DevTable& TCu = c_tabs[TC];
  const DevTable& TIt = c_tabs[TI];
  const DevTable& TSt = c_tabs[TS];
  const uint8_t* p = b.params + 128ull * r;
  uint32_t* log = tp.log + (uint64_t)r * TLOG;
  if (PH == PH_DETECT && b.nparts <= 1 && x.reorder) {  // 16 lanes, one logged slot each
    if (!active) return;
    const uint32_t row = log[sub];
    if (row == ROW_NONE) return;
    if (sub < 15) {  // same units as the general path below
      const uint32_t gq = col_group(TSt, S_QUANTITY);
      unit_w<PH>(TSt, gq, row, x);
      if (col_group(TSt, S_YTD) != gq) col_upd3<PH>(TSt, S_YTD, S_ORDER_CNT, S_REMOTE_CNT, row, x);
    } else {
      unit_a<PH>(TDi, col_group(TDi, D_NEXT_O_ID), row, x, true);
    }
    return;
  }
  if (PH == PH_DETECT && b.nparts <= 1) {
    // unpartitioned detection needs no parameters: execute logged every line slot (ROW_NONE
    // when unused) and the district row.  4 lanes per NewOrder (lanes_of), 4 log slots per
    // lane: a lane's log words and then all of their mark words are loaded together -- 8 txns
    // per warp instead of 2, and no dependent chain per unit
    if (!active) return;
    uint32_t rows[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) rows[k] = log[sub + 4 * k];  // slot sub + 4k: the 4 lanes read 16 B together
    const uint32_t gq = col_group(TSt, S_QUANTITY), gy = col_group(TSt, S_YTD);
    const uint32_t go = col_group(TSt, S_ORDER_CNT), gr = col_group(TSt, S_REMOTE_CNT);
    const uint32_t ay = col_is_add(TSt, S_YTD) ? ACC_ADD : ACC_WRITE;
    const uint32_t ao = col_is_add(TSt, S_ORDER_CNT) ? ACC_ADD : ACC_WRITE;
    const uint32_t ar = col_is_add(TSt, S_REMOTE_CNT) ? ACC_ADD : ACC_WRITE;
    uint32_t bits = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {  // same units as the general path below (unit_w / col_upd3)
      if (rows[k] == ROW_NONE || sub + 4 * k == 15) continue;
      bits |= unit_bits_lim(TSt, gq, rows[k], ACC_WRITE, x.tag);
      if (gy != gq) bits |= unit_bits_lim(TSt, gy, rows[k], ay, x.tag);
      if (go != gq && go != gy) bits |= unit_bits_lim(TSt, go, rows[k], ao, x.tag);
      if (gr != gq && gr != gy && gr != go) bits |= unit_bits_lim(TSt, gr, rows[k], ar, x.tag);
    }
    if (sub == 3 && rows[3] != ROW_NONE)  // slot 15: the district row (fetch-ADD of D_NEXT_O_ID)
      bits |= unit_bits_lim(TDi, col_group(TDi, D_NEXT_O_ID), rows[3], ACC_ADD, x.tag);
    x.bits |= bits;
    return;
  }
  if (PH == PH_EXEC && b.nparts <= 1) {
    // 4 lanes per NewOrder (lanes_of): lane q takes lines q, q+4, q+8, q+12 (lane 3: lines 3, 7,
    // 11 and the header) -- so for each k the txn's 4 lanes read 4 consecutive 8-byte line records
    // (one sector) and write 4 consecutive log slots.  A lane's line records, row lookups
    // (arithmetic on the dense W/D/C/I/S key ranges) and item-price loads are all issued before any
    // is used: 8 txns per warp instead of 2, so a warp pays the parameter -> price dependency chain
    // once for 4x the lines.
    long long amount = 0, w_tax = 0, d_tax = 0, disc = 0;
    uint32_t ua = 0;
    // line validation (k_tpcc_group reads only the 16-byte headers of unpartitioned batches):
    // item in [1, 100001], quantity in [1, 10], an existing supply warehouse, and the txn's
    // items distinct (R10) -- the 4 lanes of the txn compare their 4 items each with the 16
    // the header word and the lane's line records are loaded together (the records of slots past
    // n_lines are read -- they are inside the 128-byte block -- and ignored)
    uint32_t it[4];
    uint2 v[4];
    uint32_t h0 = 0, h1 = 0;
    if (active) {
      const uint2 h = *reinterpret_cast<const uint2*>(p);  // u16 w | u8 d | u8 n_lines | u16 c | ...
      h0 = h.x;
      h1 = h.y;
    }
#pragma unroll
    for (uint32_t k = 0; k < 4; ++k) {
      const uint32_t l = sub + 4 * k;
      v[k] = make_uint2(0, 0);
      if (active && l < 15) v[k] = *reinterpret_cast<const uint2*>(p + 8 + 8 * l);  // u32 i | u16 supply_w | u8 qty
    }
    const uint32_t n = h0 >> 24;
    // header (k_tpcc_group of an unpartitioned batch does not read it): district, line count, customer
    bool bad = active && sub == 3 &&
               ((h0 & 0xFFFFu) < 1 || (h0 & 0xFFFFu) > b.nw || ((h0 >> 16) & 0xFFu) < 1 || ((h0 >> 16) & 0xFFu) > 10 ||
                n < 1 || n > 15 || (h1 & 0xFFFFu) < 1 || (h1 & 0xFFFFu) > 3000);
#pragma unroll
    for (uint32_t k = 0; k < 4; ++k) {
      const uint32_t l = sub + 4 * k;
      if (l >= n) v[k] = make_uint2(0, 0);
      // unused slots get ids no item has (and that never collide with each other)
      it[k] = (active && l < n) ? v[k].x : 0xFFFFFFF0u - l;
      const uint32_t sw = v[k].y & 0xFFFFu, q = (v[k].y >> 16) & 0xFFu;
      if (active && l < n && (v[k].x < 1 || v[k].x > 100001 || q < 1 || q > 10 || sw < 1 || sw > b.nw)) bad = true;
    }
#ifndef LTPG_DISTINCT_PAIRS  // each lane compares its 4 items with all 16 of the txn (measured
                             // faster than the fewer-compare pair scheme below: 0.185 vs 0.190 ms
                             // execute on tpcc_c4, profiles/ab_r02_distinct.txt -- register use)
#pragma unroll
    for (uint32_t j = 0; j < 4; ++j)
#pragma unroll
      for (uint32_t m = 0; m < 4; ++m) {
        const uint32_t o = __shfl_sync(0xffffffffu, it[m], j, 4);
#pragma unroll
        for (uint32_t k = 0; k < 4; ++k)
          if (o == it[k] && 4 * j + m != 4 * sub + k) bad = true;
      }
#else
#pragma unroll
    for (uint32_t k = 1; k < 4; ++k)  // pairs inside the lane
#pragma unroll
      for (uint32_t m = 0; m < k; ++m)
        if (it[k] == it[m]) bad = true;
#pragma unroll
    for (uint32_t j = 1; j <= 2; ++j)  // pairs across lanes: partners sub+1 and sub+2 (mod 4) cover all
#pragma unroll
      for (uint32_t m = 0; m < 4; ++m) {
        const uint32_t o = __shfl_sync(0xffffffffu, it[m], (sub + j) & 3u, 4);
#pragma unroll
        for (uint32_t k = 0; k < 4; ++k)
          if (o == it[k]) bad = true;
      }
#endif
    if (bad) atomicOr(b.err, ERR_EINVAL);
    const bool warp_bad = __any_sync(0xffffffffu, bad);  // the batch is rejected: skip the work
    if (active && !warp_bad) {
      const uint32_t w = h0 & 0xFFFFu, d = (h0 >> 16) & 0xFFu, c = h1 & 0xFFFFu;
      uint32_t qt[4], ri[4], rs[4];
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint32_t l = sub + 4 * k;
        qt[k] = (v[k].y >> 16) & 0xFFu;
        ri[k] = l < n ? rowof(TIt, TI, v[k].x, x.dmask) : ROW_NONE;
        rs[k] = l < n ? rowof(TSt, TS, kS(v[k].y & 0xFFFFu, v[k].x), x.dmask) : ROW_NONE;
      }
      long long price[4];
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) price[k] = ri[k] != ROW_NONE ? rd(TIt, I_PRICE, ri[k]) : 0;
#ifndef LTPG_NO_HDR_EARLY
      // header lane: the static W / D / C reads go out with the item prices (one load wave);
      // issued after the line stores below they would wait behind them (possible aliasing)
      uint32_t row_w = ROW_NONE, row_d = ROW_NONE, row_c = ROW_NONE;
      if (sub == 3) {
        row_w = rowof(TWh, TW, w, x.dmask);
        row_d = rowof(TDi, TD, kD(w, d), x.dmask);
        row_c = rowof(TCu, TC, kC(w, d, c), x.dmask);
        if (row_w != ROW_NONE && row_d != ROW_NONE && row_c != ROW_NONE) {
          w_tax = rd(TWh, W_TAX, row_w);  // static reads: unmarked (R4)
          d_tax = rd(TDi, D_TAX, row_d);
          disc = rd(TCu, C_DISCOUNT, row_c);
        }
      }
#endif
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint32_t l = sub + 4 * k;
        if (l >= 15) continue;
        uint32_t row_s = ROW_NONE;
        if (l < n) {
          if (ri[k] == ROW_NONE) {
            ua = 1;  // unused item id: NewOrder rollback (R11)
          } else {
#ifdef LTPG_AMOUNT_IN_LOOP
            amount += (long long)qt[k] * price[k];
#endif
            row_s = rs[k];
            if (row_s == ROW_NONE) internal_error(x);
          }
        }
        log[l] = row_s;  // ROW_NONE: unused line slot
        if (row_s != ROW_NONE) {
          const uint32_t gq = col_group(TSt, S_QUANTITY);
          unit_w<PH>(TSt, gq, row_s, x);  // S_QUANTITY: conditional RMW -> WRITE unit
          if (col_group(TSt, S_YTD) != gq) col_upd3<PH>(TSt, S_YTD, S_ORDER_CNT, S_REMOTE_CNT, row_s, x);
        }
      }
      (void)it;
#ifndef LTPG_AMOUNT_IN_LOOP
      // the amounts after every mark and log store of the lane were issued: the item-price round
      // trip overlaps them instead of holding them back (price[k] == 0 for unused slots and items)
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) amount += (long long)qt[k] * price[k];
#endif
      if (sub == 3) {  // header: warehouse / district / customer reads, fetch-ADD of D_NEXT_O_ID
#ifdef LTPG_NO_HDR_EARLY
        const uint32_t row_w = rowof(TWh, TW, w, x.dmask), row_d = rowof(TDi, TD, kD(w, d), x.dmask),
                       row_c = rowof(TCu, TC, kC(w, d, c), x.dmask);
#endif
        if (row_w == ROW_NONE || row_d == ROW_NONE || row_c == ROW_NONE) {
          internal_error(x);
          log[15] = ROW_NONE;
        } else {
#ifdef LTPG_NO_HDR_EARLY
          w_tax = rd(TWh, W_TAX, row_w);  // static reads: unmarked (R4)
          d_tax = rd(TDi, D_TAX, row_d);
          disc = rd(TCu, C_DISCOUNT, row_c);
#endif
          log[15] = row_d;
          unit_a<PH>(TDi, col_group(TDi, D_NEXT_O_ID), row_d, x, true);
        }
      }
    }
    amount += __shfl_xor_sync(0xffffffffu, amount, 1);  // sums over the txn's 4 lanes
    amount += __shfl_xor_sync(0xffffffffu, amount, 2);
    ua |= __shfl_xor_sync(0xffffffffu, ua, 1);
    ua |= __shfl_xor_sync(0xffffffffu, ua, 2);
    if (active && sub == 3) {
      if (ua) b.ua[r] = 1;
      longlong2* res = reinterpret_cast<longlong2*>(b.res + 4ull * r);
      // [o_id (assigned after detection if committed), total, sum of amounts, 0]
      res[0] = make_longlong2(0, amount * (10000 - disc) * (10000 + w_tax + d_tax) / 100000000);
      res[1] = make_longlong2(amount, 0);
    }
    return;
  }
  if (PH == PH_WB && b.nparts <= 1) {
    // 4 lanes per committed NewOrder, lane q takes lines q, q+4, q+8, q+12 (the 4 lanes of a txn
    // write 4 consecutive ORDER_LINE rows per store); a lane's line records, item prices and
    // stock rows are all loaded before any is used
    uint32_t remote = 0, w = 0, d = 0, n = 0, c = 0;
    // the stock row block holds the four counters side by side (row-block layout, 32 B): read
    // and written as two 16-byte vectors instead of four 8-byte accesses to the same sector
    const bool svec = stock_block_vec(TSt);
    if (active) {
      const uint2 hh = *reinterpret_cast<const uint2*>(p);
      const uint32_t h0 = hh.x, h1 = hh.y;
      w = h0 & 0xFFFFu, d = (h0 >> 16) & 0xFFu, n = h0 >> 24, c = h1 & 0xFFFFu;
      uint2 v[4];
      uint32_t rs[4];
      long long price[4], sq[4], sy[4], so[4], sr[4];
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint32_t l = sub + 4 * k;
        v[k] = l < n ? *reinterpret_cast<const uint2*>(p + 8 + 8 * l) : make_uint2(0, 0);
        rs[k] = l < n ? log[l] : ROW_NONE;
      }
      // every stock column the lines update is read in this one wave: the stores below could
      // alias later loads, so a read-modify-write per column would serialise 3 round trips per line
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint32_t ri = sub + 4 * k < n ? rowof(TIt, TI, v[k].x, x.dmask) : ROW_NONE;
        price[k] = ri != ROW_NONE ? rd(TIt, I_PRICE, ri) : 0;  // committed: every item exists
        const bool h = rs[k] != ROW_NONE;
        if (h && svec) {
          const longlong2* sp = reinterpret_cast<const longlong2*>(col_ptr(TSt, S_QUANTITY, rs[k]));
          const longlong2 a = sp[0], bq = sp[1];
          sq[k] = a.x, sy[k] = a.y, so[k] = bq.x, sr[k] = bq.y;
        } else {
          sq[k] = h ? rd(TSt, S_QUANTITY, rs[k]) : 0;
          sy[k] = h ? rd(TSt, S_YTD, rs[k]) : 0;
          so[k] = h ? rd(TSt, S_ORDER_CNT, rs[k]) : 0;
          sr[k] = h ? rd(TSt, S_REMOTE_CNT, rs[k]) : 0;
        }
      }
      const long long o = no_oid(b, tp, r, w, d);
      const uint64_t okey = kO(w, d, (uint64_t)o);
      const DevTable& TOL_ = c_tabs[TOL];
      // append position: chunk base + in-chunk prefix of committed NewOrders (k_no_chunk); the
      // row counter is read before any store (a store could alias it and force a reload)
      const unsigned long long pref = tp.no_pref[r] + tp.chunk_tot[r >> tp.chunk_shift];
      const unsigned long long ol0 = *TOL_.n_rows;
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint32_t l = sub + 4 * k;
        if (l >= n) continue;
        const uint32_t i = v[k].x, sw = v[k].y & 0xFFFFu, qty = (v[k].y >> 16) & 0xFFu;
        const uint32_t rem = sw != w;
        remote |= rem;
        const uint32_t row_s = rs[k];
        if (row_s != ROW_NONE) {
          const long long q = sq[k];
          const long long nq = q >= (long long)qty + 10 ? q - qty : q - qty + 91;
          // the counters may be ADD columns (delayed mode), but only NewOrder touches STOCK and
          // every NewOrder writes the row's S_QUANTITY unit (WAW): this txn is the row's only
          // committed toucher in the batch (and its items are distinct, R10), so plain
          // read-modify-writes of the values read above are exact (no atomics)
          const auto add = [](long long a, long long dv) {
            return (long long)((unsigned long long)a + (unsigned long long)dv);
          };
          if (svec) {
            longlong2* sp = reinterpret_cast<longlong2*>(col_ptr(TSt, S_QUANTITY, row_s));
            sp[0] = make_longlong2(nq, add(sy[k], qty));
            sp[1] = make_longlong2(add(so[k], 1), add(sr[k], rem));
          } else {
            wr(TSt, S_QUANTITY, row_s, nq);
            wr(TSt, S_YTD, row_s, add(sy[k], qty));
            wr(TSt, S_ORDER_CNT, row_s, add(so[k], 1));
            wr(TSt, S_REMOTE_CNT, row_s, add(sr[k], rem));
          }
        }
        const uint32_t row = (uint32_t)(ol0 + (pref >> 32) + l);  // ORDER_LINE row
        wr(TOL_, OL_I_ID, row, i);
        wr(TOL_, OL_SUPPLY_W_ID, row, sw);
        wr(TOL_, OL_QUANTITY, row, qty);
        wr(TOL_, OL_AMOUNT, row, (long long)qty * price[k]);
        wr(TOL_, OL_DELIVERY_D, row, 0);
        TOL_.rowkey[row] = okey * 16 + l + 1;  // PK index entry deferred (capi.cu idx_lag)
        TOL_.valid[row] = 1;
      }
    }
    remote |= __shfl_xor_sync(0xffffffffu, remote, 1);
    remote |= __shfl_xor_sync(0xffffffffu, remote, 2);
    if (active && sub == 0) {  // ORDER and NEW_ORDER rows
      const DevTable& TOr = c_tabs[TO];
      const DevTable& TOL_ = c_tabs[TOL];
      const DevTable& TNw = c_tabs[TNO];
      const long long o = no_oid(b, tp, r, w, d);
      if (tp.oid_inline) b.res[4ull * r] = o;
      const uint64_t okey = kO(w, d, (uint64_t)o);
      const unsigned long long pref = tp.no_pref[r] + tp.chunk_tot[r >> tp.chunk_shift];
      const unsigned long long nr_o = *TOr.n_rows, nr_ol = *TOL_.n_rows, nr_no = *TNw.n_rows;  // before stores
      const long long clock = b_clock(b);
      const uint32_t orow = (uint32_t)(nr_o + (uint32_t)pref);
      if (TOr.aux) TOr.aux[orow] = (uint32_t)(nr_ol + (pref >> 32));  // contiguous lines
      wr(TOr, O_C_ID, orow, c);
      wr(TOr, O_ENTRY_D, orow, clock);
      wr(TOr, O_OL_CNT, orow, n);
      wr(TOr, O_ALL_LOCAL, orow, !remote);
      wr(TOr, O_CARRIER_ID, orow, 0);
      TOr.rowkey[orow] = okey;
      TOr.valid[orow] = 1;
      const uint32_t nrow = (uint32_t)(nr_no + (uint32_t)pref);
      wr(TNw, NO_O_ID, nrow, o);
      TNw.rowkey[nrow] = okey;
      TNw.valid[nrow] = 1;
      IdxSlot *so, *sn;
      idx_insert2(TOr, okey, so, TNw, okey, sn);
      if (so) so->row = orow; else internal_error(x);
      if (sn) sn->row = nrow; else internal_error(x);
    }
    return;
  }
  uint32_t w = 0, d = 0, n = 0, c = 0;
  if (active) {
    w = p16(p, 0);
    d = p[2];
    n = p[3];
    c = p16(p, 4);
  }
  long long amount = 0;
  uint32_t remote = 0, ua = 0;
  uint32_t i = 0, sw = 0, qty = 0, row_s = ROW_NONE;
  if (PH == PH_EXEC && active && sub < 15 && sub >= n) log[sub] = ROW_NONE;  // unused line slot
  // partitioned (§8(e)): the home partition owns the header, the order inserts and the
  // result; each stock line belongs to the owner of its supply warehouse
  const bool home = active && owns_w(b, w);
  bool line = active && sub < n;
  bool own_line = false;
  if (line) {
    const uint8_t* L = p + 8 + 8 * sub;
    i = p32(L, 0);
    sw = p16(L, 4);
    qty = L[6];
    remote = sw != w;
    own_line = owns_w(b, sw);
    line = home || own_line;
  }
  if (line) {
    if (PH == PH_EXEC || PH == PH_WB) {
      const PP pi = pp_issue(TIt, TI, i, x.dmask);  // item and stock lookups in flight together
      PP ps{};
      if (PH == PH_EXEC && own_line) ps = pp_issue(TSt, TS, kS(sw, i), x.dmask);
      const uint32_t row_i = pp_finish(TIt, pi);
      if (row_i == ROW_NONE) {
        ua = 1;  // unused item id: NewOrder rollback (R11)
      } else {
        amount = (long long)qty * rd(TIt, I_PRICE, row_i);
      }
      if (PH == PH_EXEC) {
        if (!ua && own_line) {
          row_s = pp_finish(TSt, ps);
          if (row_s == ROW_NONE) internal_error(x);
        }
        log[sub] = row_s;
      }
    }
    if (PH != PH_EXEC) {
      row_s = log[sub];
    }
    if (row_s != ROW_NONE) {
      const uint32_t gq = col_group(TSt, S_QUANTITY);
      unit_w<PH>(TSt, gq, row_s, x);  // S_QUANTITY: conditional RMW -> WRITE unit
      if (col_group(TSt, S_YTD) != gq)  // delayed mode: the counters form their own ADD unit
        col_upd3<PH>(TSt, S_YTD, S_ORDER_CNT, S_REMOTE_CNT, row_s, x);
      if (PH == PH_WB) {
        const long long q = rd(TSt, S_QUANTITY, row_s);
        wr(TSt, S_QUANTITY, row_s, q >= (long long)qty + 10 ? q - qty : q - qty + 91);
        // the counters may be ADD columns (delayed mode), but only NewOrder touches STOCK and
        // every NewOrder writes the row's S_QUANTITY unit (WAW): this txn is the row's only
        // committed toucher in the batch, so plain read-modify-writes are exact (no atomics)
        const auto inc = [&](uint32_t c, long long v) {
          long long* pc = col_ptr(TSt, c, row_s);
          *pc = (long long)((unsigned long long)*pc + (unsigned long long)v);
        };
        inc(S_YTD, qty);
        inc(S_ORDER_CNT, 1);
        inc(S_REMOTE_CNT, remote);
      }
    }
  }
  // header lane: warehouse / district / customer reads, fetch-ADD of D_NEXT_O_ID
  long long w_tax = 0, d_tax = 0, disc = 0;
  if (home && sub == 15) {
    uint32_t row_d;
    if (PH == PH_EXEC) {
      const PP pw = pp_issue(TWh, TW, w, x.dmask), pd = pp_issue(TDi, TD, kD(w, d), x.dmask),
               pc = pp_issue(TCu, TC, kC(w, d, c), x.dmask);
      const uint32_t row_w = pp_finish(TWh, pw);
      row_d = pp_finish(TDi, pd);
      const uint32_t row_c = pp_finish(TCu, pc);
      if (row_w == ROW_NONE || row_d == ROW_NONE || row_c == ROW_NONE) {
        internal_error(x);
        row_d = ROW_NONE;
      } else {
        w_tax = rd(TWh, W_TAX, row_w);  // static reads: unmarked (R4)
        d_tax = rd(TDi, D_TAX, row_d);
        disc = rd(TCu, C_DISCOUNT, row_c);
      }
      log[15] = row_d;
    } else {
      row_d = log[15];
    }
    if (row_d != ROW_NONE) unit_a<PH>(TDi, col_group(TDi, D_NEXT_O_ID), row_d, x, true);
  }
  if (PH == PH_EXEC) {
    const long long sum = seg16_sum(amount);
    ua = seg16_or(ua);
    if (active && ua && sub == 15) b.ua[r] = 1;
    if (home && sub == 15) {
      long long* res = b.res + 4ull * r;
      res[0] = 0;  // o_id: assigned after detection if committed
      res[1] = sum * (10000 - disc) * (10000 + w_tax + d_tax) / 100000000;
      res[2] = sum;
      res[3] = 0;
    }
  }
  if (PH == PH_WB) {
    const uint32_t all_local = !seg16_or(remote);
    if (home) {
      const long long o = b.res[4ull * r];
      const uint64_t okey = kO(w, d, (uint64_t)o);
      const DevTable& TOr = c_tabs[TO];
      const DevTable& TOL_ = c_tabs[TOL];
      const DevTable& TNw = c_tabs[TNO];
      // append position: chunk base + in-chunk prefix of committed NewOrders (k_no_chunk)
      const unsigned long long pref = tp.no_pref[r] + tp.chunk_tot[r / NO_CHUNK];
      if (active && sub < n) {  // ORDER_LINE row
        const uint32_t row = (uint32_t)(*TOL_.n_rows + (pref >> 32) + sub);
        wr(TOL_, OL_I_ID, row, i);
        wr(TOL_, OL_SUPPLY_W_ID, row, sw);
        wr(TOL_, OL_QUANTITY, row, qty);
        wr(TOL_, OL_AMOUNT, row, amount);
        wr(TOL_, OL_DELIVERY_D, row, 0);
        TOL_.rowkey[row] = okey * 16 + sub + 1;  // PK index entry deferred (capi.cu idx_lag)
        TOL_.valid[row] = 1;
      }
      if (sub == 15) {  // ORDER and NEW_ORDER rows
        const uint32_t orow = (uint32_t)(*TOr.n_rows + (uint32_t)pref);
        if (TOr.aux) TOr.aux[orow] = (uint32_t)(*TOL_.n_rows + (pref >> 32));  // contiguous lines
        wr(TOr, O_C_ID, orow, c);
        wr(TOr, O_ENTRY_D, orow, b_clock(b));
        wr(TOr, O_OL_CNT, orow, n);
        wr(TOr, O_ALL_LOCAL, orow, all_local);
        wr(TOr, O_CARRIER_ID, orow, 0);
        TOr.rowkey[orow] = okey;
        TOr.valid[orow] = 1;
        const uint32_t nrow = (uint32_t)(*TNw.n_rows + (uint32_t)pref);
        wr(TNw, NO_O_ID, nrow, o);
        TNw.rowkey[nrow] = okey;
        TNw.valid[nrow] = 1;
        IdxSlot *so, *sn;
        idx_insert2(TOr, okey, so, TNw, okey, sn);
        if (so) so->row = orow; else internal_error(x);
        if (sn) sn->row = nrow; else internal_error(x);
      }
    }
  }
}

// ---- Payment (TPC-C 2.5) ------------------------------------------------------------------
template <int PH>
__device__ void proc_payment(const BatchDev& b, const TpccParams& tp, uint32_t r, Tx& x, long long* agg = nullptr) {
  const DevTable& TWh = c_tabs[TW];
  const DevTable& TDi = c_tabs[TD];
  const DevTable& TCu = c_tabs[TC];
  uint32_t* log = tp.log + (uint64_t)r * TLOG;
  if (PH == PH_DETECT && b.nparts <= 1) {  // unpartitioned detection: the logged rows suffice
    const uint4 lg = *reinterpret_cast<const uint4*>(log);  // one 16-byte load (TLOG keeps rows aligned)
    col_upd<PH>(TWh, W_YTD, lg.x, x, true);
    col_upd<PH>(TDi, D_YTD, lg.y, x, true);
    col_upd3<PH>(TCu, C_BALANCE, C_YTD_PAYMENT, C_PAYMENT_CNT, lg.z, x);
    return;
  }
  // the parameter fields in two vector loads (one lane per Payment: field-by-field byte loads were
  // 7 load instructions, each touching 32 different blocks)
  const uint8_t* p = b.params + 128ull * r;
  const uint4 hv = *reinterpret_cast<const uint4*>(p);
  const uint32_t w = hv.x & 0xFFFFu, d = (hv.x >> 16) & 0xFFu, by_name = hv.x >> 24, cw = hv.y & 0xFFFFu,
                 cd = (hv.y >> 16) & 0xFFu;
  uint32_t cid = hv.z & 0xFFFFu;
  const uint32_t clast = hv.z >> 16;
  const long long amount = p64(p, 16);
  // partitioned (§8(e)): warehouse + district on the home partition, the customer (its
  // by-name lookup, result and HISTORY row) on the customer's owner
  const bool home = owns_w(b, w), cust = owns_w(b, cw);
  uint32_t row_w = ROW_NONE, row_d = ROW_NONE, row_c = ROW_NONE;
  if (PH == PH_EXEC && (w < 1 || w > b.nw || d < 1 || d > 10 || cw < 1 || cw > b.nw || cd < 1 || cd > 10 ||
                        by_name > 1 || (by_name ? clast > 999 : (cid < 1 || cid > 3000)))) {
    atomicOr(b.err, ERR_EINVAL);  // validation (k_tpcc_group of an unpartitioned batch reads no Payment)
    return;
  }
  if (PH == PH_EXEC) {
    if (cust && by_name) cid = (uint32_t)tp.by_name[kD(cw, cd) * 1000 + clast];  // static secondary index
    if (home) {  // (dense W / D keys: arithmetic; two in-flight probes (pp_issue) cost execute 16
                 // registers and spills of its slot loop for a case no TPC-C table layout hits)
      row_w = rowof(TWh, TW, w, x.dmask);
      row_d = rowof(TDi, TD, kD(w, d), x.dmask);
      if (row_w == ROW_NONE || row_d == ROW_NONE) { internal_error(x); return; }
    }
    if (cust) {
      row_c = cid ? rowof(TCu, TC, kC(cw, cd, cid), x.dmask) : ROW_NONE;
      if (row_c == ROW_NONE) { internal_error(x); return; }
      longlong2* res = reinterpret_cast<longlong2*>(b.res + 4ull * r);
      res[0] = make_longlong2(cid, col_is_add(TCu, C_BALANCE) ? 0 : rd(TCu, C_BALANCE, row_c));  // pre-image (strict only)
      res[1] = make_longlong2(0, 0);
    }
    *reinterpret_cast<uint4*>(log) = make_uint4(row_w, row_d, row_c, cid);
  } else {
    const uint4 lg = *reinterpret_cast<const uint4*>(log);
    row_w = lg.x;
    row_d = lg.y;
    row_c = lg.z;
    cid = lg.w;
  }
  if (home) {
    col_upd<PH>(TWh, W_YTD, row_w, x, true);
    col_upd<PH>(TDi, D_YTD, row_d, x, true);
  }
  if (cust) col_upd3<PH>(TCu, C_BALANCE, C_YTD_PAYMENT, C_PAYMENT_CNT, row_c, x);
  // HISTORY row inputs loaded before the balance stores (a store could alias them)
  const DevTable& THi = c_tabs[TH];  // keyless append, no marks
  unsigned long long h_tid = 0, h_rows = 0;
  if (PH == PH_WB && cust) {
    h_tid = b.tid[r];
    h_rows = *THi.n_rows;
  }
  if (PH == PH_WB && home) {
    if (agg) {  // block-aggregated delayed adds (k_tpcc_phase)
      atomicAdd(reinterpret_cast<unsigned long long*>(agg + w), (unsigned long long)amount);
      if (tp.agg_dsz)
        atomicAdd(reinterpret_cast<unsigned long long*>(agg + tp.nw + 1 + kD(w, d)), (unsigned long long)amount);
      else
        addv(TDi, D_YTD, row_d, amount);
    } else {
      addv(TWh, W_YTD, row_w, amount);
      addv(TDi, D_YTD, row_d, amount);
    }
  }
  if (PH == PH_WB && cust) {
    addv(TCu, C_BALANCE, row_c, -amount);
    addv(TCu, C_YTD_PAYMENT, row_c, amount);
    addv(TCu, C_PAYMENT_CNT, row_c, 1);
    // warp-aggregated append: one counter atomic per warp (every committed Payment appends;
    // per-lane atomics on the single counter serialised), consecutive rows per warp
    const uint32_t am = __activemask(), lane = threadIdx.x & 31, lead = __ffs(am) - 1;
    uint32_t hb = 0;
    if (lane == lead) hb = atomicAdd(tp.misc + M_HIST, (uint32_t)__popc(am));
    hb = __shfl_sync(am, hb, lead) + __popc(am & ((1u << lane) - 1u));
    const uint32_t row = (uint32_t)(h_rows + hb);
    wr(THi, H_C_ID, row, cid);
    wr(THi, H_C_D_ID, row, cd);
    wr(THi, H_C_W_ID, row, cw);
    wr(THi, H_D_ID, row, d);
    wr(THi, H_W_ID, row, w);
    wr(THi, H_DATE, row, b_clock(b));
    wr(THi, H_AMOUNT, row, amount);
    wr(THi, H_TID, row, (long long)h_tid);
    wr(THi, H_SEQ, row, 0);
    THi.valid[row] = 1;
  }
}

// ---- OrderStatus (TPC-C 2.6) with a predefined order key ----------------------------
// 4 lanes per txn (8 txns per warp): lane 3 finds the customer and its order, then lane q reads
// order lines 4q..4q+3 (all of a lane's line loads in flight together).
template <int PH>
__device__ void proc_orderstatus(const BatchDev& b, const TpccParams& tp, uint32_t r, uint32_t sub, bool active,
                                 Tx& x) {  // (active: by value -- a txn failing validation stops here)
  const DevTable& TCu = c_tabs[TC];
  const DevTable& TOr = c_tabs[TO];
  const DevTable& TOL_ = c_tabs[TOL];
  const uint8_t* p = b.params + 128ull * r;
  uint32_t* log = tp.log + (uint64_t)r * TLOG;
  uint32_t w = 0, d = 0, cid = 0, o = 0, cnt = 0, row_c = ROW_NONE, row_o = ROW_NONE;
  long long bal = 0, carrier = 0;
  if (active) {
    w = p16(p, 0);
    d = p[2];
  }
  if (active && sub == 3 && PH == PH_EXEC &&
      (w < 1 || w > b.nw || d < 1 || d > 10 || p[3] > 1 || (p[3] ? p16(p, 6) > 999 : (p16(p, 4) < 1 || p16(p, 4) > 3000)))) {
    atomicOr(b.err, ERR_EINVAL);  // validation (k_tpcc_group of an unpartitioned batch reads no OrderStatus)
    active = false;
  }
  if (active && sub == 3) {
    if (PH == PH_EXEC) {
      cid = p[3] ? (uint32_t)tp.by_name[kD(w, d) * 1000 + p16(p, 6)] : p16(p, 4);
      row_c = cid ? rowof(TCu, TC, kC(w, d, cid), x.dmask) : ROW_NONE;
      if (row_c != ROW_NONE) {
        bal = rd(TCu, C_BALANCE, row_c);
        o = (uint32_t)rd(TCu, C_INIT_O_ID, row_c);
        row_o = probe(TOr, kO(w, d, o));
      }
      if (row_o == ROW_NONE) {
        internal_error(x);
      } else {
        carrier = rd(TOr, O_CARRIER_ID, row_o);
        cnt = (uint32_t)rd(TOr, O_OL_CNT, row_o);
      }
      log[15] = row_c;
      log[16] = row_o;
    } else {
      row_c = log[15];
      row_o = log[16];
      cnt = row_o != ROW_NONE ? (uint32_t)rd(TOr, O_OL_CNT, row_o) : 0;
    }
    if (row_c != ROW_NONE) unit_r<PH>(TCu, col_group(TCu, C_BALANCE), row_c, x);
    if (row_o != ROW_NONE) unit_r<PH>(TOr, col_group(TOr, O_CARRIER_ID), row_o, x);
  }
  uint32_t olrow = (PH == PH_EXEC && active && sub == 3 && row_o != ROW_NONE && TOr.aux) ? TOr.aux[row_o] : ROW_NONE;
  o = __shfl_sync(0xffffffffu, o, 3, 4);
  cnt = __shfl_sync(0xffffffffu, cnt, 3, 4);
  olrow = __shfl_sync(0xffffffffu, olrow, 3, 4);
  long long dd = 0;
  uint32_t row_ol[4];
#pragma unroll
  for (uint32_t k = 0; k < 4; ++k) {  // the lane's line rows: from ORDER.aux (contiguous) or probed
    const uint32_t l = sub + 4 * k;  // the txn's 4 lanes: 4 consecutive lines per k
    row_ol[k] = ROW_NONE;
    if (!active || l >= cnt || l >= 15) continue;
    if (PH == PH_EXEC) {
      row_ol[k] = olrow != ROW_NONE ? olrow + l : probe(TOL_, kO(w, d, o) * 16 + l + 1);
      if (row_ol[k] == ROW_NONE) internal_error(x);
      log[l] = row_ol[k];
    } else {
      row_ol[k] = log[l];
    }
  }
#pragma unroll
  for (uint32_t k = 0; k < 4; ++k) {
    if (row_ol[k] == ROW_NONE) continue;
    if (PH == PH_EXEC) dd += rd(TOL_, OL_DELIVERY_D, row_ol[k]);
    unit_r<PH>(TOL_, col_group(TOL_, OL_DELIVERY_D), row_ol[k], x);
  }
  if (PH == PH_EXEC) {
    dd += __shfl_xor_sync(0xffffffffu, dd, 1);  // sum over the txn's 4 lanes
    dd += __shfl_xor_sync(0xffffffffu, dd, 2);
    if (active && sub == 3) {
      long long* res = b.res + 4ull * r;
      res[0] = cid;
      res[1] = bal;
      res[2] = carrier;
      res[3] = dd;
    }
  }
}

// ---- Delivery (TPC-C 2.7), rows re-derived in every phase -----------------------------------
// Shared per warehouse: every Delivery RMWs the cursors of all ten districts of its warehouse
// (WRITE units), so of a warehouse's Deliveries in a batch only the smallest rank can commit
// (R1 and NEXT-1: WAW aborts).  They all read the same snapshot -- same cursors, orders, lines
// and customers -- so they mark the same units, where the smallest rank's mark is the minimum,
// and return the same results (the carrier is not part of them).  Only that rank (dl_min[w],
// from k_tpcc_group) executes, marks and is checked; the others copy its result slots and take
// the WAW verdict.  Result-identical to running each one (oracle parity).
// The phase kernel runs the leaders by warehouse (slot type SL_DLW: one 16-lane slot per
// warehouse with a Delivery in the batch, lane d-1 = district d), and detection visits every
// Delivery txn once more with one lane each (SL_DLT) to give the followers their verdict and
// results -- the followers, nearly all Deliveries, cost one load each instead of a 16-lane slot.

// one district of leader txn x.r (lane d - 1)
template <int PH>
__device__ void delivery_district(const BatchDev& b, uint32_t w, uint32_t d, long long carrier, Tx& x,
                                  long long& delivered, long long& total) {
  const DevTable& TDi = c_tabs[TD];
  const DevTable& TCu = c_tabs[TC];
  const DevTable& TOr = c_tabs[TO];
  const DevTable& TOL_ = c_tabs[TOL];
  const DevTable& TNw = c_tabs[TNO];
  const uint32_t row_d = rowof(TDi, TD, kD(w, d), x.dmask);
  if (row_d == ROW_NONE) {
    internal_error(x);
    return;
  }
  const long long o = rd(TDi, D_NEXT_DELIV_O_ID, row_d);
  unit_w<PH>(TDi, col_group(TDi, D_NEXT_DELIV_O_ID), row_d, x, true);  // RMW of the cursor
  const uint64_t nok = kO(w, d, (uint64_t)o);
  uint64_t hn_, ho_;
  const ulonglong2 vn = probe_issue(TNw, nok, hn_), vo = probe_issue(TOr, nok, ho_);  // together
  if (PH == PH_DETECT && x.done()) return;  // conflict already found: the verdict cannot change
  const uint32_t row_no = probe_finish(TNw, nok, hn_, vn);
  if (row_no == ROW_NONE) {
    // queue empty in S: READ of the D_NEXT_O_ID unit (same-batch NewOrders conflict)
    unit_r<PH>(TDi, col_group(TDi, D_NEXT_O_ID), row_d, x, true);
    return;
  }
  // every Delivery of a warehouse in the batch reads the same cursor and so delivers the same
  // order: its NEW_ORDER / ORDER / ORDER_LINE / CUSTOMER units are as hot as the district's
  // (E >> 1) -- marks take the read-before-atomicMin filter
  for (uint32_t g = 0; g < TNw.n_groups; ++g) unit_w<PH>(TNw, g, row_no, x, true);  // DELETE
  const uint32_t row_o = probe_finish(TOr, nok, ho_, vo);
  if (row_o == ROW_NONE) {
    internal_error(x);
    return;
  }
  unit_w<PH>(TOr, col_group(TOr, O_CARRIER_ID), row_o, x, true);
  const uint32_t cid = (uint32_t)rd(TOr, O_C_ID, row_o);
  const uint32_t cnt = (uint32_t)rd(TOr, O_OL_CNT, row_o);
  long long sum = 0;
  uint32_t row_ol[15];
  const uint32_t olrow = TOr.aux ? TOr.aux[row_o] : ROW_NONE;  // lines are contiguous rows
#pragma unroll
  for (uint32_t l = 0; l < 15; ++l)  // otherwise all order-line probes in flight together
    row_ol[l] = l < cnt ? (olrow != ROW_NONE ? olrow + l : probe(TOL_, nok * 16 + l + 1)) : ROW_NONE;
  const uint32_t row_c = rowof(TCu, TC, kC(w, d, cid), x.dmask);
#pragma unroll
  for (uint32_t l = 0; l < 15; ++l) {
    if (l >= cnt) continue;
    if (row_ol[l] == ROW_NONE) { internal_error(x); continue; }
    unit_w<PH>(TOL_, col_group(TOL_, OL_DELIVERY_D), row_ol[l], x, true);
    sum += rd(TOL_, OL_AMOUNT, row_ol[l]);
    if (PH == PH_WB) wr(TOL_, OL_DELIVERY_D, row_ol[l], b_clock(b));
  }
  if (row_c == ROW_NONE) {
    internal_error(x);
  } else {
    col_upd3<PH>(TCu, C_BALANCE, C_DELIVERY_CNT, C_DELIVERY_CNT, row_c, x, true);
    if (PH == PH_WB) {
      addv(TCu, C_BALANCE, row_c, sum);
      addv(TCu, C_DELIVERY_CNT, row_c, 1);
    }
  }
  if (PH == PH_WB) {
    wr(TOr, O_CARRIER_ID, row_o, carrier);
    TNw.valid[row_no] = 0;
    IdxSlot* sl = idx_slot(TNw, nok);
    if (sl) sl->row = ROW_NONE;
    wr(TDi, D_NEXT_DELIV_O_ID, row_d, o + 1);
  }
  delivered = 1;
  total = sum;
}

// the leader of warehouse w (slot type SL_DLW, 16 lanes: lane d-1 = district d); r = dl_min[w]
template <int PH>
__device__ void proc_delivery(const BatchDev& b, uint32_t r, uint32_t sub, bool active, Tx& x) {
  long long delivered = 0, total = 0;
  const uint8_t* p = b.params + 128ull * r;
  if (active && sub < 10) delivery_district<PH>(b, p16(p, 0), sub + 1, p[2], x, delivered, total);
  if (PH == PH_EXEC) {
    delivered = seg16_sum(delivered);
    total = seg16_sum(total);
    if (active && sub == 0) {
      long long* res = b.res + 4ull * r;
      res[0] = delivered;
      res[1] = total;
      res[2] = 0;
      res[3] = 0;
    }
  }
}
// detection pass over every Delivery txn (slot type SL_DLT, one lane each): a follower (not its
// warehouse's smallest rank) takes the WAW verdict and copies the leader's results; returns
// whether r is a follower (a leader's verdict comes from its SL_DLW slot)
__device__ __forceinline__ bool delivery_follower(const BatchDev& b, const TpccParams& tp, uint32_t r, Tx& x) {
  const uint32_t rmin = tp.dl_min[p16(b.params + 128ull * r, 0)];
  if (rmin == r) return false;
  x.bits |= CF_WAW;  // WAW on the district cursors against rank rmin < r
  long long* res = b.res + 4ull * r;  // written by rmin's execute
  const long long* src = b.res + 4ull * rmin;
  res[0] = src[0];
  res[1] = src[1];
  res[2] = src[2];
  res[3] = src[3];
  return true;
}

// ---- StockLevel (TPC-C 2.8): shared per district ---------------------------------------------
// Every StockLevel of a district reads the same snapshot: D_NEXT_O_ID, the last 20 orders, their
// distinct items and those items' S_QUANTITY.  So the window is evaluated once per district with
// StockLevels in the batch (one warp each) into a prefix table low[t] = #distinct items with
// S_QUANTITY < t (t = 0..256); a txn's result is low[threshold].  Its read set is the district's
// unit set, so its RAW test (R1: any smaller rank wrote/added a unit) reduces to one comparison
// with M = the smallest mark rank over that set.  Result- and verdict-identical to one warp per
// txn; the work drops from per-txn to per-district (~66x at 64 warehouses, 2^20 txns).
constexpr int SL_SLOTS = 20 * 15;
constexpr int SL_HASH = 512;
constexpr int SL_T = 257;

__device__ __forceinline__ uint32_t sl_dk_of(const BatchDev& b, uint32_t r) {
  const uint8_t* p = b.params + 128ull * r;
  return (uint32_t)kD(p16(p, 0), p[2]);
}

// every StockLevel: minimum rank per district; the first one lists the district
__global__ void __launch_bounds__(256) k_sl_claim(BatchDev b, TpccParams tp, SlScratch sl) {
  if (*b.err) return;
  const uint32_t n = tp.counts[4];
  const uint32_t* list = tp.list + 4ull * tp.max_txns;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint32_t r = list[i];
    const uint32_t dk = sl_dk_of(b, r);
    if (atomicMin(sl.minr + dk, r) == 0xFFFFFFFFu) {
      const uint32_t idx = atomicAdd(sl.cnt, 1u);
      sl.dk[idx] = dk;
      sl.slot[dk] = idx;
    }
  }
}

// one warp per listed district: window, distinct items, S_QUANTITY prefix table; NEXT-1 minR
__device__ __forceinline__ void sl_district_body(const BatchDev& b, const SlScratch& sl, uint32_t vb, uint32_t nvb) {
  if (*(volatile uint32_t*)b.err) return;
  __shared__ uint32_t items_s[8][SL_SLOTS];
  __shared__ uint32_t set_s[8][SL_HASH];
  __shared__ uint32_t hist_s[8][SL_T + 1];
  const DevTable& TDi = c_tabs[TD];
  const DevTable& TOr = c_tabs[TO];
  const DevTable& TOL_ = c_tabs[TOL];
  const DevTable& TSt = c_tabs[TS];
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  uint32_t* items = items_s[wib];
  uint32_t* set = set_s[wib];
  uint32_t* hist = hist_s[wib];
  const uint32_t dmask = *b.dense_live;
  const bool reorder = b.flags & LTPG_FLAG_REORDER;
  const uint32_t nd_total = *(volatile uint32_t*)sl.cnt;
  const uint32_t nwarps = nvb * (blockDim.x >> 5);
  for (uint32_t idx = vb * (blockDim.x >> 5) + wib; idx < nd_total; idx += nwarps) {
    const uint32_t dk = sl.dk[idx];
    uint32_t w = dk / 10, d = dk % 10;
    if (d == 0) { d = 10; w -= 1; }  // kD(w, 10) == kD(w + 1, 0)
    const uint32_t row_d = rowof(TDi, TD, dk, dmask);
    if (row_d == ROW_NONE) {
      if (lane == 0) atomicOr(b.err, ERR_EINTERNAL);
      continue;
    }
    const long long nx = rd(TDi, D_NEXT_O_ID, row_d);
    for (uint32_t s2 = lane; s2 < SL_SLOTS; s2 += 32) items[s2] = 0;
    for (uint32_t s2 = lane; s2 < SL_HASH; s2 += 32) set[s2] = 0;
    for (uint32_t s2 = lane; s2 <= SL_T; s2 += 32) hist[s2] = 0;
    __syncwarp();
    if (lane < 20) {
      const long long o = nx - 20 + lane;
      const uint32_t row_o = probe(TOr, kO(w, d, (uint64_t)o));
      if (row_o == ROW_NONE) {
        atomicOr(b.err, ERR_EINTERNAL);
      } else {
        const uint32_t cnt = (uint32_t)rd(TOr, O_OL_CNT, row_o);  // static
        const uint32_t olrow = TOr.aux ? TOr.aux[row_o] : ROW_NONE;  // lines are contiguous rows
        uint32_t row_ol[15];
#pragma unroll
        for (uint32_t l = 0; l < 15; ++l)  // otherwise independent probes issued back to back
          row_ol[l] = l < cnt ? (olrow != ROW_NONE ? olrow + l : probe(TOL_, kO(w, d, (uint64_t)o) * 16 + l + 1))
                              : ROW_NONE;
#pragma unroll
        for (uint32_t l = 0; l < 15; ++l)
          if (l < cnt) {
            if (row_ol[l] == ROW_NONE) atomicOr(b.err, ERR_EINTERNAL);
            else items[lane * 15 + l] = (uint32_t)rd(TOL_, OL_I_ID, row_ol[l]);  // static
          }
      }
    }
    __syncwarp();
    // distinct items: the first inserter of an item into the shared-memory set appends it to a
    // compact list (the slot array is reused: items were consumed into registers first)
    constexpr uint32_t MAXU = (SL_SLOTS + 31) / 32;
    uint32_t mine[MAXU];
#pragma unroll
    for (uint32_t u = 0; u < MAXU; ++u) {
      const uint32_t j = lane + 32 * u;
      mine[u] = j < SL_SLOTS ? items[j] : 0u;
    }
    __syncwarp();
    uint32_t nd = 0;
#pragma unroll
    for (uint32_t u = 0; u < MAXU; ++u) {
      const uint32_t it = mine[u];
      bool first = false;
      if (it) {
        uint32_t h = (it * 2654435761u) >> 23;  // 9 bits
        for (;;) {
          const uint32_t old = atomicCAS(set + h, 0u, it);
          if (old == 0u) { first = true; break; }
          if (old == it) break;
          h = (h + 1) & (SL_HASH - 1);
        }
      }
      const uint32_t m = __ballot_sync(0xffffffffu, first);
      if (first) items[nd + __popc(m & ((1u << lane) - 1))] = it;
      nd += __popc(m);
    }
    __syncwarp();
    // stock rows and quantities of the distinct items (dense key -> row: no index access)
    uint32_t rows[MAXU];
#pragma unroll
    for (uint32_t u = 0; u < MAXU; ++u) {
      const uint32_t j = lane + 32 * u;
      rows[u] = j < nd ? rowof(TSt, TS, kS(w, items[j]), dmask) : ROW_NONE;
    }
    long long q[MAXU];
#pragma unroll
    for (uint32_t u = 0; u < MAXU; ++u) q[u] = rows[u] != ROW_NONE ? rd(TSt, S_QUANTITY, rows[u]) : 0;
    const mark_t rtag = epoch_tag(b_epoch(b)) | grank_of(b, sl.minr[dk]);
    const uint32_t gq = col_group(TSt, S_QUANTITY);
#pragma unroll
    for (uint32_t u = 0; u < MAXU; ++u) {
      const uint32_t j = lane + 32 * u;
      if (j >= nd) continue;
      if (rows[u] == ROW_NONE) { atomicOr(b.err, ERR_EINTERNAL); continue; }
      sl.rows[(uint64_t)idx * SL_SLOTS + j] = rows[u];
      // bucket q + 1 (clamped): q < t  <=>  bucket <= t
      const long long bq = q[u] + 1 < 0 ? 0 : (q[u] + 1 > SL_T ? SL_T : q[u] + 1);
      atomicAdd(hist + bq, 1u);
      if (reorder && TSt.rmarks) mark_unit(TSt, MK_R, gq, rows[u], rtag, true);  // NEXT-1 minR
    }
    if (lane == 0 && reorder && TDi.rmarks)
      mark_unit(TDi, MK_R, col_group(TDi, D_NEXT_O_ID), row_d, rtag, true);
    __syncwarp();
    // low[t] = sum of hist[0..t]: 9 buckets per lane, then a warp scan of the lane sums
    constexpr uint32_t PER = (SL_T + 31) / 32;
    uint32_t v[PER], run = 0;
#pragma unroll
    for (uint32_t k = 0; k < PER; ++k) {
      const uint32_t t = lane * PER + k;
      run += t < SL_T ? hist[t] : 0u;
      v[k] = run;
    }
    uint32_t incl = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= (uint32_t)o) incl += y;
    }
    const uint32_t base = incl - run;
#pragma unroll
    for (uint32_t k = 0; k < PER; ++k) {
      const uint32_t t = lane * PER + k;
      if (t < SL_T) sl.low[(uint64_t)idx * SL_T + t] = base + v[k];
    }
    if (lane == 0) {
      sl.nx[idx] = nx;
      sl.nd[idx] = nd;
      sl.rowd[idx] = row_d;
    }
    __syncwarp();
  }
}
__global__ void __launch_bounds__(256) k_sl_district(BatchDev b, SlScratch sl) {
  sl_district_body(b, sl, blockIdx.x, gridDim.x);
}

// detection, one warp per listed district: M = smallest write / add rank over its unit set
__device__ __forceinline__ void sl_detect_body(const BatchDev& b, const SlScratch& sl, uint32_t vb, uint32_t nvb) {
  if (*(volatile uint32_t*)b.err) return;
  const DevTable& TDi = c_tabs[TD];
  const DevTable& TSt = c_tabs[TS];
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t nd_total = *(volatile uint32_t*)sl.cnt;
  const uint32_t nwarps = nvb * (blockDim.x >> 5);
  const uint32_t gq = col_group(TSt, S_QUANTITY), gd = col_group(TDi, D_NEXT_O_ID);
  for (uint32_t idx = vb * (blockDim.x >> 5) + wib; idx < nd_total; idx += nwarps) {
    const uint32_t nd = sl.nd[idx];
    uint32_t m = 0xFFFFFFFFu;
    auto wa = [&](const DevTable& T, uint32_t g, uint32_t row) {
      const uint32_t w = mark_rank(*wmark_ptr(T, g, row), b_epoch(b));
      const uint32_t a = ((T.add_groups >> g) & 1u) ? mark_rank(*amark_ptr(T, g, row), b_epoch(b)) : 0xFFFFFFFFu;
      return w < a ? w : a;
    };
    if (lane == 0) m = wa(TDi, gd, sl.rowd[idx]);
    for (uint32_t j = lane; j < nd; j += 32) m = min(m, wa(TSt, gq, sl.rows[(uint64_t)idx * SL_SLOTS + j]));
    m = __reduce_min_sync(0xffffffffu, m);
    if (lane == 0) sl.m[idx] = m;
  }
}
__global__ void __launch_bounds__(256) k_sl_detect(BatchDev b, SlScratch sl) { sl_detect_body(b, sl, blockIdx.x, gridDim.x); }

// per StockLevel txn: result from the district's table, RAW verdict from its M
__device__ __forceinline__ void sl_txn_body(const BatchDev& b, const TpccParams& tp, const SlScratch& sl, uint32_t vb,
                                            uint32_t nvb) {
  if (*(volatile uint32_t*)b.err) return;
  const uint32_t n = *(volatile const uint32_t*)(tp.counts + 4);
  const uint32_t* list = tp.list + 4ull * tp.max_txns;
  const bool reorder = b.flags & LTPG_FLAG_REORDER;
  for (uint32_t i = vb * blockDim.x + threadIdx.x; i < n; i += nvb * blockDim.x) {
    const uint32_t r = list[i];
    const uint8_t* p = b.params + 128ull * r;
    const uint32_t idx = sl.slot[kD(p16(p, 0), p[2])];
    long long* res = b.res + 4ull * r;
    res[0] = sl.low[(uint64_t)idx * SL_T + p[3]];
    res[1] = sl.nx[idx];
    res[2] = 0;
    res[3] = 0;
    // NEXT-1: read-only procedures never abort under reordering
    const uint32_t flag = (!reorder && sl.m[idx] < grank_of(b, r) ? CF_RAW : 0u) | (b.ua[r] ? CF_UA : 0u);
    if (b.nparts > 1) b.lflag[r] = (uint8_t)flag;
    else b.status[r] = status_of_bits(flag, reorder);
  }
}
__global__ void __launch_bounds__(256) k_sl_txn(BatchDev b, TpccParams tp, SlScratch sl) {
  sl_txn_body(b, tp, sl, blockIdx.x, gridDim.x);
}

// ---- the phase kernel: type-homogeneous warps over the per-type txn lists -------------------------

// TMASK: procedure types this launch runs.  StockLevel (32 lanes, 26 KB of shared memory per
// block, many registers) runs in its own launch so it does not cap the occupancy of the
// others -- each type group gets its own launch configuration.
constexpr uint32_t TM_MAIN = 0x0Fu;
// Warp slot types of the phase kernel: the procedure types 0..4 (Delivery's type 3 is the
// detection-only pass over every Delivery txn) and SL_DLW, the Delivery leader of a warehouse.
constexpr uint32_t SL_DLT = 3, SL_DLW = 5, NSLOT = 6;
// lanes per slot: Payment 1; Delivery txn pass 1; Delivery leader 16 (one per district);
// OrderStatus 4 (4 lines per lane); StockLevel 32 (k_sl_*); NewOrder 16 -- 4 in execution and detection of an unpartitioned
// batch (4 lines / units per lane, see proc_neworder; execute 0.255 -> 0.198 ms, detect 0.113 ->
// 0.087 ms on tpcc_c4) except detection under NEXT-1 reordering, where every unit's three marks
// are read and 16 lanes measured faster
__device__ __forceinline__ uint32_t lanes_of(uint32_t t, int PH, uint32_t nparts, bool reorder) {
  return t == 1 || t == SL_DLT ? 1u
                          : (t == 4 ? 32u
                                    : (t == 2 || (t == 0 && nparts <= 1 && (PH != PH_DETECT || !reorder)) ? 4u : 16u));
}  // NewOrder, Payment, OrderStatus, Delivery (StockLevel: k_sl_*)
// minimum resident blocks per phase (register cap): detection is a chain of dependent
// loads (params -> log -> marks) and gains most from occupancy (measured: 8 -> 32 regs);
// write-back keeps every stock column of a lane's lines in registers (one load wave instead of
// a read-modify-write chain per column): 3 blocks / 80 regs, 0.165 -> 0.138 ms on tpcc_c4
// (4 blocks / 64 regs: 0.141; 6 blocks / 40 regs spilled: 0.170)
#ifndef LTPG_EXEC_MINB
#define LTPG_EXEC_MINB 4
#endif
#ifndef LTPG_DETECT_MINB
#define LTPG_DETECT_MINB 8
#endif
#ifndef LTPG_WB_MINB
#define LTPG_WB_MINB 3
#endif
// the phase body over (virtual) blocks vb of nvb; FUSED (single-launch path): the write-back's
// row-counter advance is left to the caller
template <int PH, uint32_t TMASK, bool FUSED>
__device__ __forceinline__ void tpcc_phase_body(const BatchDev& b, const TpccParams& tp, uint32_t vb, uint32_t nvb) {
  const bool reorder = b.flags & LTPG_FLAG_REORDER;
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  // warp slots by procedure type.  Detection: the longest chains first (OrderStatus, Delivery,
  // NewOrder, Payment), so that the grid's tail is made of short Payment warps (0.088 -> 0.077
  // ms on tpcc_c4); execute keeps the type order (measured slower the other way round)
  // write-back starts with the Delivery leaders (their chains -- cursor, NEW_ORDER, ORDER, lines,
  // customer per district -- are the longest; last, they were the grid's tail: tpcc_c4 write-back
  // 0.122 -> 0.115 ms, profiles/ab_r02_bar_detect.txt); execute keeps the type order (neutral)
  constexpr uint32_t ORD = PH == PH_DETECT ? (2u | SL_DLW << 4 | 0u << 8 | SL_DLT << 12 | 1u << 16 | 4u << 20)
                           : PH == PH_WB   ? (SL_DLW | 0u << 4 | 1u << 8 | 2u << 12 | SL_DLT << 16 | 4u << 20)
                                           : (0u | 1u << 4 | 2u << 8 | SL_DLW << 12 | SL_DLT << 16 | 4u << 20);  // slot j -> type
  // One read of the error word per block (the kernel has block barriers, and the word can be
  // raised by other blocks of this grid while this one starts), issued together with the list
  // lengths: slot counts and warp-slot prefixes per slot type, in shared memory (computed once
  // per block; as register arrays they cost every thread 12 registers for the whole kernel)
  __shared__ uint32_t s_err, cnt[NSLOT], pre[NSLOT + 1];
  const uint32_t dmask = *b.dense_live;  // procedures never insert into / delete from W, D, C, I, S
  if (threadIdx.x == 0) {
    uint32_t c5[NTYPES];
#pragma unroll
    for (int t = 0; t < NTYPES; ++t) c5[t] = (TMASK >> t) & 1u ? tp.counts[t] : 0u;
    s_err = *(volatile uint32_t*)b.err;
    pre[0] = 0;
#pragma unroll
    for (int j = 0; j < NSLOT; ++j) {
      const uint32_t t = (ORD >> (4 * j)) & 15u;
      const bool on = (TMASK >> (t == SL_DLW ? SL_DLT : t)) & 1u;
      cnt[j] = !on ? 0u : (t == SL_DLW ? tp.nw : (t == SL_DLT && PH != PH_DETECT ? 0u : c5[t]));
      const uint32_t lp = 5 - (__ffs(lanes_of(t, PH, b.nparts, reorder)) - 1);  // log2(txns per warp slot)
      pre[j + 1] = pre[j] + ((cnt[j] + (1u << lp) - 1) >> lp);
    }
  }
  __syncthreads();
  if (s_err) return;  // (write-back: the row counters then stay put -- no last block runs)
  // ECAPACITY before anything is written back: the grouping counts are final here (a block
  // barrier + fence + counter per grouping block for a "last block" cost 22% of that kernel)
  if (PH == PH_EXEC && TMASK == TM_MAIN && vb == 0 && threadIdx.x == 0) tpcc_capacity_tail(b, tp);
  // write-back with delayed W_YTD / D_YTD (ADD columns): the block's committed Payments add
  // into shared-memory deltas per warehouse (and district), flushed with one atomic per touched
  // row at the end -- hundreds of thousands of same-row atomics at the L2 become a few per block
  extern __shared__ long long agg[];
  const bool aggw = PH == PH_WB && col_is_add(c_tabs[TW], W_YTD) && col_is_add(c_tabs[TD], D_YTD);
  if (aggw) {
    for (uint32_t i = threadIdx.x; i < tp.nw + 1 + tp.agg_dsz; i += blockDim.x) agg[i] = 0;
    __syncthreads();
  }
  // execute: shared-memory marks of the hot WAREHOUSE / DISTRICT units (hot_mark)
  mark_t* hm = (PH == PH_EXEC && tp.hot_words) ? reinterpret_cast<mark_t*>(agg) : nullptr;
  if (hm) {
    for (uint32_t i = threadIdx.x; i < tp.hot_words; i += blockDim.x) hm[i] = 0xFFFFFFFFu;
    __syncthreads();
  }
  const uint32_t nwarps = nvb * (blockDim.x >> 5);
  // warp slot w -> slot type t, this lane's list position k and sub-lane (warp-uniform type)
  const auto decode = [&](uint32_t w, uint32_t& t, uint32_t& k, uint32_t& sub, uint32_t& ct) {
    uint32_t j = 0, lw = w;
    ct = cnt[0];
#pragma unroll
    for (int jj = 1; jj < NSLOT; ++jj)
      if (w >= pre[jj]) { j = jj; lw = w - pre[jj]; ct = cnt[jj]; }
    t = (ORD >> (4 * j)) & 15u;
    const uint32_t ll = __ffs(lanes_of(t, PH, b.nparts, reorder)) - 1;  // lanes per txn: a power of two
    k = (lw << (5 - ll)) + (lane >> ll);
    sub = lane & ((1u << ll) - 1u);
  };
  // the list entry of a warp's NEXT slot is loaded before the current slot runs: the list ->
  // parameters -> rows chain of each slot starts one load later than its list read
  const auto list_entry = [&](uint32_t w) -> uint32_t {
    uint32_t t, k, sub, ct;
    decode(w, t, k, sub, ct);
    return (t != SL_DLW && k < ct) ? tp.list[(uint64_t)t * tp.max_txns + k] : 0u;
  };
  uint32_t w = vb * (blockDim.x >> 5) + wib;
  uint32_t r_next = w < pre[NSLOT] ? list_entry(w) : 0u;
  for (; w < pre[NSLOT]; w += nwarps) {
    uint32_t t, k, sub, ct;
    decode(w, t, k, sub, ct);
    const uint32_t L = lanes_of(t, PH, b.nparts, reorder);
    bool active = k < ct;
#ifdef LTPG_NO_PREFETCH
    uint32_t r = list_entry(w);
#else
    uint32_t r = r_next;
    if (w + nwarps < pre[NSLOT]) r_next = list_entry(w + nwarps);
#endif
    if (t == SL_DLW) {  // warehouse k + 1's Delivery leader (write-back: only if it committed)
      r = active ? tp.dl_min[k + 1] : ~0u;
      active = r != ~0u && (PH != PH_WB || b.status[r] == LTPG_ST_COMMIT);
      if (!active) r = 0;
    } else if (!active) {
      r = 0;
    }
    const uint32_t gr = active ? grank_of(b, r) : 0u;  // conflict TID (global rank of a sharded batch)
    Tx x{dmask, gr, b_epoch(b), epoch_tag(b_epoch(b)) | gr, !(b.flags & LTPG_FLAG_NO_MARK_FILTER), 0u, b.err, reorder,
         hm, tp.nw};
    bool go = active;  // write-back runs over the committed re-list (k_tpcc_relist) only
    bool status_here = true;  // detection: this slot decides txn r's verdict
    // NEXT-1: read-only procedures (OrderStatus, StockLevel) can never abort under reordering
    if (PH == PH_DETECT && reorder && (t == 2 || t == 4)) go = false;
    switch (t) {
      case 0: proc_neworder<PH>(b, tp, r, sub, go, x); break;
      case 1: if (go) proc_payment<PH>(b, tp, r, x, aggw ? agg : nullptr); break;
      case 2: if (PH != PH_WB) proc_orderstatus<PH>(b, tp, r, sub, go, x); break;
      case SL_DLW: proc_delivery<PH>(b, r, sub, go, x); break;
      case SL_DLT: if (go && PH == PH_DETECT) status_here = delivery_follower(b, tp, r, x); break;
      default:
        break;  // StockLevel: shared per district (k_sl_*)
    }
    if (PH == PH_DETECT) {  // per-txn OR of the conflict bits over the txn's lanes
      const uint32_t seg = L == 32 ? 0xffffffffu : (((1u << L) - 1u) << (lane & ~(L - 1u)));
      const uint32_t bw = __ballot_sync(0xffffffffu, x.bits & CF_WAW) & seg;
      const uint32_t br = __ballot_sync(0xffffffffu, x.bits & CF_RAW) & seg;
      const uint32_t bx = __ballot_sync(0xffffffffu, x.bits & CF_WAR) & seg;
      if (active && sub == 0 && status_here) {
        const uint32_t flag = (bw ? CF_WAW : 0u) | (br ? CF_RAW : 0u) | (bx ? CF_WAR : 0u) | (b.ua[r] ? CF_UA : 0u);
        if (b.nparts > 1) b.lflag[r] = (uint8_t)flag;  // partitioned: exchanged before write-back
        else b.status[r] = status_of_bits(flag, reorder);
      }
    }
  }
  if (hm) {  // flush: one global atomicMin per unit this block marked
    __syncthreads();
    const DevTable& TWh = c_tabs[TW];
    const DevTable& TDi = c_tabs[TD];
    for (uint32_t i = threadIdx.x; i < tp.nw; i += blockDim.x) {  // WAREHOUSE group 0
      const mark_t v = hm[i];
      if (v != 0xFFFFFFFFu) atomicMin((TWh.add_groups & 1u) ? amark_ptr(TWh, 0, i) : wmark_ptr(TWh, 0, i), v);
    }
#pragma unroll
    for (uint32_t g = 0; g < 3; ++g) {  // DISTRICT groups 0..2
      const mark_t* hg = hm + tp.nw + g * 10 * tp.nw;
      const bool add = (TDi.add_groups >> g) & 1u;
      for (uint32_t row = threadIdx.x; row < 10 * tp.nw; row += blockDim.x) {
        const mark_t v = hg[row];
        if (v != 0xFFFFFFFFu) atomicMin(add ? amark_ptr(TDi, g, row) : wmark_ptr(TDi, g, row), v);
      }
    }
  }
  if (aggw) {
    __syncthreads();
    const DevTable& TWh = c_tabs[TW];
    const DevTable& TDi = c_tabs[TD];
    for (uint32_t i = threadIdx.x; i < tp.nw + 1 + tp.agg_dsz; i += blockDim.x) {
      const long long v = agg[i];
      if (!v) continue;
      const bool isw = i <= tp.nw;
      const DevTable& T = isw ? TWh : TDi;
      const uint32_t row = rowof(T, isw ? TW : TD, isw ? i : i - tp.nw - 1, dmask);
      if (row == ROW_NONE) { atomicOr(b.err, ERR_EINTERNAL); continue; }
      addv(T, isw ? W_YTD : D_YTD, row, v);
    }
  }
  if (!FUSED && PH == PH_WB && TMASK == TM_MAIN && last_block(tp.misc + M_DONE_WB) && threadIdx.x == 0)
    tpcc_advance_tail(b, tp);
}
template <int PH, uint32_t TMASK>
#ifndef LTPG_EXEC_THREADS
#define LTPG_EXEC_THREADS 256
#endif
__global__ void __launch_bounds__(PH == PH_EXEC ? LTPG_EXEC_THREADS : 256,
                                  (PH == PH_EXEC ? LTPG_EXEC_MINB * 256 / LTPG_EXEC_THREADS
                                                 : PH == PH_DETECT ? LTPG_DETECT_MINB : LTPG_WB_MINB))
    k_tpcc_phase(BatchDev b, TpccParams tp) {
  tpcc_phase_body<PH, TMASK, false>(b, tp, blockIdx.x, gridDim.x);
}

// ---- K-tgroup: validation + per-type lists (warp-aggregated appends) ----------------------------
// FULL (partitioned batches): the whole 128-byte block is parsed here -- a NewOrder's supply
// warehouses decide whether it touches this partition.  Otherwise (one partition) only the
// first 16 bytes of each block are read: every field but the NewOrder lines sits there, and the
// lines are validated by execute, which reads them anyway (proc_neworder; an invalid line
// raises ERR_EINVAL there, before anything is written back).  134 -> 16 MB read per 2^20 txns.
// CLAIM (single-launch path, !FULL): k_sl_claim folded in -- a StockLevel's district is claimed
// here (smallest rank per district, the first claimer lists it).  vb: the (virtual) block index.
template <bool FULL, bool CLAIM>
__device__ __forceinline__ void tpcc_group_body(const BatchDev& b, const TpccParams& tp, uint32_t vb,
                                                const SlScratch& sl) {
  // FULL: the warp's 32 parameter blocks (4 KB, contiguous) staged through shared memory with
  // coalesced 16-byte loads; each lane then parses its own block.  Rows are padded to 33
  // words: with a 128-byte stride every lane's field would sit in the same bank (32-way
  // conflicts measured at 45% short-scoreboard stalls)
  constexpr uint32_t SROW = 132;
  __shared__ __align__(16) uint8_t stage[FULL ? 8 : 1][FULL ? 32 * SROW : 16];
  const uint32_t r = vb * blockDim.x + threadIdx.x;
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t r0 = r - lane;
  uint8_t* sw = stage[FULL ? wib : 0];
  uint4 head = make_uint4(0, 0, 0, 0);  // !FULL: the block's first 16 bytes, in registers
  if (FULL) {
#pragma unroll
    for (uint32_t k = 0; k < 8; ++k) {
      const uint32_t c = k * 32 + lane;  // 16-byte chunk of the warp's 4 KB
      if (r0 + c / 8 < b.n_txns) {
        const uint4 v = *reinterpret_cast<const uint4*>(b.params + 128ull * r0 + 16 * c);
        uint32_t* d = reinterpret_cast<uint32_t*>(sw + SROW * (c / 8) + 16 * (c % 8));
        d[0] = v.x;
        d[1] = v.y;
        d[2] = v.z;
        d[3] = v.w;
      }
    }
    __syncwarp();
  }
  uint32_t t = 0xFF, lines = 0;
  bool bad = false;
  if (r < b.n_txns) {
    if (r > 0 && b.tid[r] <= b.tid[r - 1]) bad = true;
    if (b.grank && (b.grank[r] >= b.n_global || (r > 0 && b.grank[r] <= b.grank[r - 1]))) bad = true;
    t = b.ptype[r];
    // !FULL: only Delivery and StockLevel blocks are read here (their warehouse / district index
    // per-batch scratch before execute runs); NewOrder, Payment and OrderStatus are validated by
    // execute, which reads their parameters anyway -- so this kernel streams the 9 bytes of TID and
    // type per txn instead of fetching every 128-byte block (its first 16 bytes cost a whole line)
    if (!FULL && (t == 3 || t == 4)) head = *reinterpret_cast<const uint4*>(b.params + 128ull * r);
    const uint8_t* p = FULL ? sw + SROW * lane : reinterpret_cast<const uint8_t*>(&head);
    const uint32_t W = tp.nw;
    auto okw = [W](uint32_t w) { return w >= 1 && w <= W; };
    auto okd = [](uint32_t d) { return d >= 1 && d <= 10; };
    if ((FULL || t == 3 || t == 4) && !okw(p16(p, 0))) bad = true;
    if (!FULL && t <= 2) {
      lines = t == 0 ? 15 : 0;  // capacity: a NewOrder may append up to 15 lines (its count is checked in execute)
    } else switch (t) {
      case 0: {
        const uint32_t nl = p[3], c = p16(p, 4);
        if (!okd(p[2]) || nl < 1 || nl > 15 || c < 1 || c > 3000) { bad = true; break; }
        lines = nl;
        if (!FULL) break;  // lines: validated by execute
        uint32_t it[15];
#pragma unroll
        for (uint32_t l = 0; l < 15; ++l) {
          const uint8_t* L = p + 8 + 8 * l;
          it[l] = l < nl ? p32(L, 0) : 0xFFFFFFF0u - l;  // unused slots never collide
          if (l < nl && (!okw(p16(L, 4)) || L[6] < 1 || L[6] > 10 || it[l] < 1 || it[l] > 100001)) bad = true;
        }
#pragma unroll
        for (uint32_t l = 1; l < 15; ++l)
#pragma unroll
          for (uint32_t m = 0; m < l; ++m)
            if (it[l] == it[m]) bad = true;  // R10: distinct items (registers, unrolled)
        break;
      }
      case 1:
        if (!okd(p[2]) || !okw(p16(p, 4)) || !okd(p[6]) || p[3] > 1) bad = true;
        else if (p[3] ? p16(p, 10) > 999 : (p16(p, 8) < 1 || p16(p, 8) > 3000)) bad = true;
        break;
      case 2:
        if (!okd(p[2]) || p[3] > 1) bad = true;
        else if (p[3] ? p16(p, 6) > 999 : (p16(p, 4) < 1 || p16(p, 4) > 3000)) bad = true;
        break;
      case 3:
        if (p[2] < 1 || p[2] > 10) bad = true;
        break;
      case 4:
        if (!okd(p[2])) bad = true;
        break;
      default:
        bad = true;
    }
    if (bad) atomicOr(b.err, ERR_EINVAL);
  }
  // partitioned (§8(e)): list the txn only where it touches owned rows; count the appends
  // this partition may make (ORDER/NEW_ORDER/ORDER_LINE at home, HISTORY at the customer)
  bool touch = false;
  uint32_t no_home = 0, pay_cust = 0;
  if (r < b.n_txns && !bad) {
    const uint8_t* p = FULL ? sw + SROW * lane : reinterpret_cast<const uint8_t*>(&head);
    const bool home = FULL ? owns_w(b, p16(p, 0)) : true;
    touch = home;
    // partitions the txn touches (bit q; the sharded exchange needs them, world <= 32)
    const auto pbit = [&](uint32_t w) { const uint32_t q = part_of_w(w, b.nw, b.nparts); return q < 32 ? 1u << q : 0u; };
    uint32_t pm = pbit(p16(p, 0));
    if (!FULL) {  // one partition: every txn is home; NewOrder and Payment may append
      touch = true;
      no_home = t == 0;
      pay_cust = t == 1;
    } else if (t == 0) {
      for (uint32_t l = 0; l < lines; ++l) pm |= pbit(p16(p + 8 + 8 * l, 4));
      touch = (pm >> b.part) & 1u;
      no_home = home;
      if (!home) lines = 0;
    } else if (t == 1) {
      pm |= pbit(p16(p, 4));
      pay_cust = owns_w(b, p16(p, 4));
      touch = touch || pay_cust;
    }
    if (FULL && b.pmask) b.pmask[r] = pm;
  } else {
    lines = 0;
  }
  if (t == 3 && touch) {  // smallest Delivery rank per warehouse (shared Delivery, proc_delivery)
    uint32_t* m = tp.dl_min + (FULL ? p16(sw + SROW * lane, 0) : (head.x & 0xFFFFu));
    if (r < *m) atomicMin(m, r);
  }
  if (CLAIM && !FULL && t == 4 && touch) {  // StockLevel: the district's smallest rank (k_sl_claim)
    const uint32_t dk = (uint32_t)kD(head.x & 0xFFFFu, (head.x >> 16) & 0xFFu);
    if (atomicMin(sl.minr + dk, r) == 0xFFFFFFFFu) {
      const uint32_t idx = atomicAdd(sl.cnt, 1u);
      sl.dk[idx] = dk;
      sl.slot[dk] = idx;
    }
  }
  // block-aggregated counters and per-type list positions (one atomic per block and list)
  // slots 0..4: the per-type list flags (b.kcount), 5..7: misc[M_NO_LINES], misc[M_PAY],
  // misc[M_NO]; every slot but the line count is a 0/1 flag (ballot scans), one barrier pair
  uint32_t cnt[NTYPES + 3], base[NTYPES + 3];
#pragma unroll
  for (uint32_t k = 0; k < NTYPES; ++k) cnt[k] = (t == k && !bad && touch) ? 1u : 0u;
  cnt[NTYPES] = lines;
  cnt[NTYPES + 1] = pay_cust;
  cnt[NTYPES + 2] = no_home;
  block_reserve<NTYPES + 3, ((1u << NTYPES) - 1u) | (3u << (NTYPES + 1)), NTYPES>(cnt, b.kcount, base,
                                                                                   tp.misc + M_NO_LINES);
#pragma unroll
  for (uint32_t k = 0; k < NTYPES; ++k)
    if (cnt[k]) tp.list[(uint64_t)k * tp.max_txns + base[k]] = r;
}
template <bool FULL>
__global__ void __launch_bounds__(256) k_tpcc_group(BatchDev b, TpccParams tp) {
  tpcc_group_body<FULL, false>(b, tp, blockIdx.x, SlScratch{});
}

// Unpartitioned batches: the same validation and lists with 4 consecutive txns per thread (their
// TID, type and -- Delivery / StockLevel only -- 16-byte heads issued together): a quarter of the
// blocks, each paying the load -> reservation -> list-store chain once for 4 txns (one txn per
// thread left every block a chain of dependent round trips: 3.5 waves of them at 2^20 txns;
// measured: tpcc_c5 grouping 17 -> 14.5 us, tpcc_c4 unchanged at 22 us).
// List order inside a type list is free (lists only assign txns to warp slots).
__global__ void __launch_bounds__(256) k_tpcc_group4(BatchDev b, TpccParams tp) {
  constexpr uint32_t G4 = 4;
  const uint32_t r0 = (blockIdx.x * blockDim.x + threadIdx.x) * G4;
  const uint32_t W = tp.nw;
  auto okw = [W](uint32_t w) { return w >= 1 && w <= W; };
  auto okd = [](uint32_t d) { return d >= 1 && d <= 10; };
  unsigned long long tid[G4 + 1];
  uint32_t ty[G4];
  uint4 head[G4];
#pragma unroll
  for (uint32_t j = 0; j < G4; ++j) {
    const uint32_t r = r0 + j;
    tid[j + 1] = r < b.n_txns ? b.tid[r] : 0ull;
    ty[j] = r < b.n_txns ? b.ptype[r] : 0xFFu;
  }
  tid[0] = (r0 > 0 && r0 < b.n_txns) ? b.tid[r0 - 1] : 0ull;
#pragma unroll
  for (uint32_t j = 0; j < G4; ++j) {
    head[j] = make_uint4(0, 0, 0, 0);
    if (ty[j] == 3 || ty[j] == 4) head[j] = *reinterpret_cast<const uint4*>(b.params + 128ull * (r0 + j));
  }
  // slots 0..4: per-type list counts (b.kcount), 5..7: misc[M_NO_LINES], misc[M_PAY], misc[M_NO]
  uint32_t cnt[NTYPES + 3], base[NTYPES + 3];
#pragma unroll
  for (uint32_t k = 0; k < NTYPES + 3; ++k) cnt[k] = 0;
  bool any_bad = false;
  uint32_t okm = 0;  // bit j: txn r0 + j is listed
#pragma unroll
  for (uint32_t j = 0; j < G4; ++j) {
    const uint32_t r = r0 + j;
    if (r >= b.n_txns) continue;
    const uint32_t t = ty[j];
    const uint8_t* p = reinterpret_cast<const uint8_t*>(&head[j]);
    bool bad = r > 0 && tid[j + 1] <= tid[j];
    if (b.grank && (b.grank[r] >= b.n_global || (r > 0 && b.grank[r] <= b.grank[r - 1]))) bad = true;
    if (t == 3) bad |= !okw(p16(p, 0)) || p[2] < 1 || p[2] > 10;
    else if (t == 4) bad |= !okw(p16(p, 0)) || !okd(p[2]);
    else if (t > 4) bad = true;
    // NewOrder / Payment / OrderStatus heads: validated by execute (which reads them anyway)
    any_bad |= bad;
    if (bad) continue;
    okm |= 1u << j;
#pragma unroll
    for (uint32_t k = 0; k < NTYPES; ++k) cnt[k] += t == k;
    cnt[NTYPES] += t == 0 ? 15u : 0u;  // capacity: a NewOrder may append up to 15 lines
    cnt[NTYPES + 1] += t == 1;
    cnt[NTYPES + 2] += t == 0;
    if (t == 3) {  // smallest Delivery rank per warehouse (shared Delivery, proc_delivery)
      uint32_t* m = tp.dl_min + (head[j].x & 0xFFFFu);
      if (r < *m) atomicMin(m, r);
    }
  }
  if (any_bad) atomicOr(b.err, ERR_EINVAL);
  block_reserve<NTYPES + 3, 0u, NTYPES>(cnt, b.kcount, base, tp.misc + M_NO_LINES);
#pragma unroll
  for (uint32_t j = 0; j < G4; ++j) {
    if (!((okm >> j) & 1u)) continue;
    const uint32_t t = ty[j];
#pragma unroll
    for (uint32_t k = 0; k < NTYPES; ++k)
      if (t == k) tp.list[(uint64_t)k * tp.max_txns + base[k]++] = r0 + j;
  }
}

// committed entries of every per-type list -> clist (order inside a list is irrelevant)
__global__ void __launch_bounds__(256) k_tpcc_relist(BatchDev b, TpccParams tp) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t pre[NTYPES + 1];
  pre[0] = 0;
#pragma unroll
  for (int t = 0; t < NTYPES; ++t) pre[t + 1] = pre[t] + b.kcount[t];
  uint32_t t = NTYPES, r = 0;
#pragma unroll
  for (int k = 0; k < NTYPES; ++k)
    if (!*b.err && i >= pre[k] && i < pre[k + 1]) {
      t = k;
      r = tp.list[(uint64_t)k * tp.max_txns + (i - pre[k])];
    }
  uint32_t cnt[NTYPES], base[NTYPES];
#pragma unroll
  for (int k = 0; k < NTYPES; ++k) cnt[k] = (t == (uint32_t)k && b.status[r] == LTPG_ST_COMMIT) ? 1u : 0u;
  block_reserve<NTYPES, (1u << NTYPES) - 1u>(cnt, tp.misc + M_CCOUNT, base);
#pragma unroll
  for (int k = 0; k < NTYPES; ++k)
    if (cnt[k]) tp.clist[(uint64_t)k * tp.max_txns + base[k]] = r;
}

// ---- NewOrder o_id: fetch-ADD pre-image = snapshot D_NEXT_O_ID + #committed NewOrders of the
//      same district with a smaller rank (P:241 prefix sum; R12) -------------------------------
// One block per NO_CHUNK ranks (4 consecutive ranks per thread): committed NewOrders of this
// partition -> their district histogram (chunk_cnt), the in-chunk exclusive prefix of
// (lines << 32 | 1) in rank order (no_pref; write-back adds the chunk base) and the chunk
// total (chunk_tot; scanned by the last block of k_no_colscan).
// RELIST (unpartitioned batches, where every txn touches this partition): also the committed
// re-list of k_tpcc_relist, from the same status reads.
// (StockLevel txns are not re-listed: write-back has nothing to do for them, and on the
// single-launch path their verdicts are written concurrently with this pass)
template <bool RELIST>
__device__ __forceinline__ void no_chunk_body(const BatchDev& b, const TpccParams& tp, uint32_t chunk, uint32_t* hist) {
  __shared__ unsigned long long wsum[8];
  if (*(volatile uint32_t*)b.err) return;
  for (uint32_t i = threadIdx.x; i < tp.dsz; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t r0 = chunk * NO_CHUNK + 4 * threadIdx.x;
  unsigned long long v[4], tsum = 0;
  uint32_t dk[4], ty[4], cm[4];
#pragma unroll
  for (uint32_t j = 0; j < 4; ++j) {
    const uint32_t r = r0 + j;
    ty[j] = r < b.n_txns ? b.ptype[r] : 0xFFu;
    cm[j] = r < b.n_txns && ty[j] != 4 && b.status[r] == LTPG_ST_COMMIT;
  }
  if (RELIST) {
    uint32_t cnt[NTYPES], base[NTYPES];
#pragma unroll
    for (uint32_t k = 0; k < NTYPES; ++k) cnt[k] = 0;
#pragma unroll
    for (uint32_t j = 0; j < 4; ++j)
#pragma unroll
      for (uint32_t k = 0; k < NTYPES; ++k) cnt[k] += (cm[j] && ty[j] == k) ? 1u : 0u;
    block_reserve<NTYPES>(cnt, tp.misc + M_CCOUNT, base);
#pragma unroll
    for (uint32_t j = 0; j < 4; ++j)
#pragma unroll
      for (uint32_t k = 0; k < NTYPES; ++k)
        if (cm[j] && ty[j] == k) tp.clist[(uint64_t)k * tp.max_txns + base[k]++] = r0 + j;
  }
#pragma unroll
  for (uint32_t j = 0; j < 4; ++j) {
    const uint32_t r = r0 + j;
    bool c = ty[j] == 0 && cm[j];
    uint32_t hdr = 0;
    if (c) {
      hdr = *reinterpret_cast<const uint32_t*>(b.params + 128ull * r);  // u16 w | u8 d | u8 n_lines
      c = owns_w(b, hdr & 0xFFFFu);
    }
    v[j] = c ? ((unsigned long long)(hdr >> 24) << 32 | 1ull) : 0ull;
    dk[j] = c ? (uint32_t)kD(hdr & 0xFFFFu, (hdr >> 16) & 0xFFu) : ~0u;
    if (c) atomicAdd(hist + dk[j], 1u);
    tsum += v[j];
  }
  unsigned long long x = tsum;  // block-wide exclusive scan of the per-thread sums, rank order
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  if (lane == 31) wsum[wib] = x;
  __syncthreads();
  unsigned long long before = 0, total = 0;
#pragma unroll
  for (uint32_t w = 0; w < 8; ++w) {
    if (w < wib) before += wsum[w];
    total += wsum[w];
  }
  unsigned long long ex = before + x - tsum;
#pragma unroll
  for (uint32_t j = 0; j < 4; ++j) {
    const uint32_t r = r0 + j;
    if (r < b.n_txns) {
      tp.no_pref[r] = ex;
      tp.dk_of[r] = dk[j];
    }
    ex += v[j];
  }
  if (threadIdx.x == 0) tp.chunk_tot[chunk] = total;
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < tp.dsz; i += blockDim.x) tp.chunk_cnt[cc_at(tp, i, chunk)] = hist[i];
  __syncthreads();  // (hist is reused by the caller's next chunk)
}
template <bool RELIST>
__global__ void __launch_bounds__(256) k_no_chunk(BatchDev b, TpccParams tp) {
  extern __shared__ uint32_t hist[];
  no_chunk_body<RELIST>(b, tp, blockIdx.x, hist);
}

// Single-launch path: the same per-chunk quantities for 32-rank chunks, one (virtual) block of
// 256 ranks = 8 chunks, one thread per rank: committed re-lists (block-aggregated), each warp's
// district counts (every district's word of the chunk, zeros included, district-major for the
// column scan's coalesced rows), the in-chunk rank among the district's committed NewOrders (dk_of: write-back adds it
// to the district's chunk base, no assignment pass) and the in-chunk prefix of (lines << 32 | 1).
__device__ __forceinline__ void no_chunk32_body(const BatchDev& b, const TpccParams& tp, uint32_t vb) {
  if (*(volatile uint32_t*)b.err) return;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t r = vb * blockDim.x + threadIdx.x, c = r >> 5;
  const uint32_t ty = r < b.n_txns ? b.ptype[r] : 0xFFu;
  const bool cm = r < b.n_txns && ty != 4 && b.status[r] == LTPG_ST_COMMIT;
  uint32_t cnt[NTYPES], base[NTYPES];
#pragma unroll
  for (uint32_t k = 0; k < NTYPES; ++k) cnt[k] = (cm && ty == k) ? 1u : 0u;
  block_reserve<NTYPES, (1u << NTYPES) - 1u>(cnt, tp.misc + M_CCOUNT, base);
#pragma unroll
  for (uint32_t k = 0; k < NTYPES; ++k)
    if (cnt[k]) tp.clist[(uint64_t)k * tp.max_txns + base[k]] = r;
  bool no = cm && ty == 0;
  uint32_t hdr = 0;
  if (no) hdr = *reinterpret_cast<const uint32_t*>(b.params + 128ull * r);  // u16 w | u8 d | u8 n_lines
  const uint32_t dk = no ? (uint32_t)kD(hdr & 0xFFFFu, (hdr >> 16) & 0xFFu) : ~0u;
  const uint32_t m = __match_any_sync(0xffffffffu, dk);
  if (c * 32 < b.n_txns) {  // district-major: [dk][chunk] (the column scan reads whole rows)
    for (uint32_t i = lane; i < tp.dsz; i += 32) tp.chunk_cnt[cc_at(tp, i, c)] = 0;
    __syncwarp();
    if (no && lane == (uint32_t)(__ffs(m) - 1)) tp.chunk_cnt[cc_at(tp, dk, c)] = __popc(m);
  }
  if (r < b.n_txns) tp.dk_of[r] = no ? __popc(m & ((1u << lane) - 1u)) : 0u;
  const unsigned long long v = no ? ((unsigned long long)(hdr >> 24) << 32 | 1ull) : 0ull;
  unsigned long long x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  if (r < b.n_txns) tp.no_pref[r] = x - v;
  if (lane == 31 && c * 32 < b.n_txns) tp.chunk_tot[c] = x;
}

// chunk totals -> exclusive chunk bases (in place) and the batch total in no_pref[n]
__device__ void chunk_total_scan(const BatchDev& b, const TpccParams& tp) {
  __shared__ unsigned long long wsum[8];
  const uint32_t nc = tp.n_chunks, per = (nc + blockDim.x - 1) / blockDim.x;
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t c0 = threadIdx.x * per;
  unsigned long long tsum = 0;
#pragma unroll 4
  for (uint32_t c = c0; c < c0 + per && c < nc; ++c) tsum += tp.chunk_tot[c];
  unsigned long long x = tsum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  if (lane == 31) wsum[wib] = x;
  __syncthreads();
  unsigned long long ex = x - tsum, total = 0;
  for (uint32_t w = 0; w < (blockDim.x >> 5); ++w) {
    if (w < wib) ex += wsum[w];
    total += wsum[w];
  }
  for (uint32_t c = c0; c < c0 + per && c < nc; ++c) {
    const unsigned long long t = tp.chunk_tot[c];
    tp.chunk_tot[c] = ex;
    ex += t;
  }
  if (threadIdx.x == 0) tp.no_pref[b.n_txns] = total;
}

// Exclusive prefix over chunks of one district's row of chunk counts (district-major, in place):
// lane l holds chunks t0 + 32 k + l of a 1024-chunk tile (coalesced loads and stores), 32 warp
// scans per tile with a running carry.  Returns the district's total.
__device__ __forceinline__ uint32_t chunk_row_scan(uint32_t* row, uint32_t nc) {
  const uint32_t lane = threadIdx.x & 31;
  uint32_t carry = 0;
  for (uint32_t t0 = 0; t0 < nc; t0 += 1024) {
    uint32_t v[32];
#pragma unroll
    for (uint32_t k = 0; k < 32; ++k) v[k] = t0 + k * 32 + lane < nc ? row[t0 + k * 32 + lane] : 0u;
#pragma unroll
    for (uint32_t k = 0; k < 32; ++k) {
      if (t0 + k * 32 >= nc) break;  // (warp-uniform)
      uint32_t x = v[k];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (uint32_t)o) x += y;
      }
      if (t0 + k * 32 + lane < nc) row[t0 + k * 32 + lane] = carry + x - v[k];
      carry += __shfl_sync(0xffffffffu, x, 31);
    }
  }
  return carry;
}

// Column scan of chunk_cnt ([district][chunk] -> exclusive prefix over chunks, in place), plus
// the district bases and the final D_NEXT_O_ID: one warp per district key.  SNAP (single-launch
// path): the caller checked the error word and dist_base already holds every district's snapshot
// D_NEXT_O_ID (read in the previous stage by the otherwise idle a8 block).
// vb of nvb = (dsz + 7) / 8 + 1 blocks (the last one scans the chunk totals).
template <bool SNAP>
__device__ __forceinline__ void no_colscan_body(const BatchDev& b, const TpccParams& tp, uint32_t vb, uint32_t nvb) {
  if (!SNAP && *(volatile uint32_t*)b.err) return;
  if (vb == nvb - 1) {  // the extra last block: chunk bases
    chunk_total_scan(b, tp);
    return;
  }
  const uint32_t dk = vb * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const uint32_t lane = threadIdx.x & 31;
  if (dk >= tp.dsz) return;
  uint32_t run_all = 0;
  if (tp.cc_dm) {
    run_all = chunk_row_scan(tp.chunk_cnt + (uint64_t)dk * tp.n_chunks, tp.n_chunks);
  } else {  // chunk-major: a column walk, 32 chunks per lane held in registers, 1024 per pass
    constexpr uint32_t PER = 32;
    for (uint32_t base = 0; base < tp.n_chunks; base += 32 * PER) {
      uint32_t v[PER];
#pragma unroll
      for (uint32_t k = 0; k < PER; ++k) {  // lane owns chunks base + [lane*PER, lane*PER+PER): loads in flight
        const uint32_t ch = base + lane * PER + k;
        v[k] = ch < tp.n_chunks ? tp.chunk_cnt[(uint64_t)ch * tp.dsz + dk] : 0u;
      }
      uint32_t tot = 0;
#pragma unroll
      for (uint32_t k = 0; k < PER; ++k) tot += v[k];
      uint32_t x = tot;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (uint32_t)o) x += y;
      }
      uint32_t run = run_all + x - tot;  // exclusive prefix of this lane's first chunk
      run_all += __shfl_sync(0xffffffffu, x, 31);
#pragma unroll
      for (uint32_t k = 0; k < PER; ++k) {
        const uint32_t ch = base + lane * PER + k;
        if (ch < tp.n_chunks) tp.chunk_cnt[(uint64_t)ch * tp.dsz + dk] = run;
        run += v[k];
      }
    }
  }
  if (!run_all || lane) return;
  const DevTable& TDi = c_tabs[TD];
  const uint32_t row_d = rowof(TDi, TD, dk, *b.dense_live);
  if (row_d == ROW_NONE) {
    atomicOr(b.err, ERR_EINTERNAL);
    return;
  }
  if (!SNAP) tp.dist_base[dk] = rd(TDi, D_NEXT_O_ID, row_d);
  addv(TDi, D_NEXT_O_ID, row_d, run_all);  // final value: snapshot + committed NewOrders (delayed add)
}
__global__ void __launch_bounds__(256) k_no_colscan(BatchDev b, TpccParams tp) {
  no_colscan_body<false>(b, tp, blockIdx.x, gridDim.x);
}

// Column scan for many districts (tpcc_c5: 5131 district keys): 8 districts per block, tiles of
// 1024 chunks x 8 districts move through shared memory with coalesced 32-byte rows, then warp w
// scans district dk0+w across the tile (k_no_colscan's one-sector-per-lane column reads: 59 us at
// 512 warehouses, 0.500 -> 0.472 ms write-back; at 64 warehouses the direct column walk is 3 us
// faster, so the launcher picks by district count)
constexpr uint32_t CS_TILE = 1024;
__global__ void __launch_bounds__(256) k_no_colscan_tiled(BatchDev b, TpccParams tp) {
  if (*b.err) return;
  if (blockIdx.x == gridDim.x - 1) {  // the extra last block: chunk bases
    chunk_total_scan(b, tp);
    return;
  }
  __shared__ uint32_t tile[CS_TILE * 9];  // [chunk][8 districts + 1 pad word]
  const uint32_t dk0 = blockIdx.x * 8, nc = tp.n_chunks;
  const uint32_t wib = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t dk = dk0 + wib;
  uint32_t run_all = 0;
  for (uint32_t t0 = 0; t0 < nc; t0 += CS_TILE) {
    const uint32_t tn = min(CS_TILE, nc - t0);
    constexpr uint32_t PER = CS_TILE * 8 / 256;  // 32 loads per thread, all in flight
    uint32_t v[PER];
#pragma unroll
    for (uint32_t k = 0; k < PER; ++k) {
      const uint32_t i = threadIdx.x + k * 256, ch = i >> 3, d = i & 7;
      v[k] = ch < tn && dk0 + d < tp.dsz ? tp.chunk_cnt[(uint64_t)(t0 + ch) * tp.dsz + dk0 + d] : 0u;
    }
#pragma unroll
    for (uint32_t k = 0; k < PER; ++k) {
      const uint32_t i = threadIdx.x + k * 256;
      tile[(i >> 3) * 9 + (i & 7)] = v[k];
    }
    __syncthreads();
    for (uint32_t c0 = 0; c0 < tn; c0 += 32) {
      const uint32_t ch = c0 + lane;
      const uint32_t v = ch < tn ? tile[ch * 9 + wib] : 0u;
      uint32_t x = v;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (uint32_t)o) x += y;
      }
      if (ch < tn) tile[ch * 9 + wib] = run_all + x - v;
      run_all += __shfl_sync(0xffffffffu, x, 31);
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < tn * 8; i += blockDim.x) {
      const uint32_t ch = i >> 3, d = i & 7;
      if (dk0 + d < tp.dsz) tp.chunk_cnt[(uint64_t)(t0 + ch) * tp.dsz + dk0 + d] = tile[ch * 9 + d];
    }
    __syncthreads();
  }
  if (dk >= tp.dsz) return;
  if (!run_all || lane) return;
  const DevTable& TDi = c_tabs[TD];
  const uint32_t row_d = rowof(TDi, TD, dk, *b.dense_live);
  if (row_d == ROW_NONE) {
    atomicOr(b.err, ERR_EINTERNAL);
    return;
  }
  const long long base = rd(TDi, D_NEXT_O_ID, row_d);
  tp.dist_base[dk] = base;
  addv(TDi, D_NEXT_O_ID, row_d, run_all);  // final value: snapshot + committed NewOrders (delayed add)
}

// one warp per chunk, ranks in order; cntd: the warp's dsz shared-memory words, each district's
// next o_id (snapshot D_NEXT_O_ID + committed NewOrders of smaller rank in earlier chunks: the
// walk below then touches shared memory only -- with the district base read from global memory
// in the walk, every step waited for an L2 round trip)
__device__ __forceinline__ void no_assign_body(const BatchDev& b, const TpccParams& tp, uint32_t chunk, long long* cntd) {
  if (*(volatile uint32_t*)b.err) return;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t r0 = chunk * NO_CHUNK;
  uint32_t dks[NO_CHUNK / 32];
#pragma unroll
  for (uint32_t it = 0; it < NO_CHUNK / 32; ++it) {  // all of the chunk's loads in flight first
    const uint32_t r = r0 + it * 32 + lane;
    dks[it] = r < b.n_txns ? tp.dk_of[r] : ~0u;
  }
  // Many districts (> COLSCAN_TILED_DSZ keys, chunk-major): only the districts of the chunk's
  // committed NewOrders (a few dozen of the 5131 at 512 warehouses; tpcc_c5 write-back 0.432 ->
  // 0.411 ms).  Otherwise the whole row (district-major gathers / one coalesced row; tpcc_c4
  // write-back 0.132 (per-district) -> 0.124 ms, profiles/ab_r02_assign.txt).  (A lane writing a
  // district another lane writes too stores the same value; dist_base of a district without
  // commits is never read.)
  if (tp.dsz > COLSCAN_TILED_DSZ) {
#pragma unroll
    for (uint32_t it = 0; it < NO_CHUNK / 32; ++it)
      if (dks[it] != ~0u) cntd[dks[it]] = tp.dist_base[dks[it]] + tp.chunk_cnt[cc_at(tp, dks[it], chunk)];
  } else {
    for (uint32_t i = lane; i < tp.dsz; i += 32) cntd[i] = tp.dist_base[i] + tp.chunk_cnt[cc_at(tp, i, chunk)];
  }
  __syncwarp();
#pragma unroll
  for (uint32_t it = 0; it < NO_CHUNK / 32; ++it) {
    const uint32_t r = r0 + it * 32 + lane;
    const uint32_t dk = dks[it];
    if (!__any_sync(0xffffffffu, dk != ~0u)) continue;
    const uint32_t m = __match_any_sync(0xffffffffu, dk);
    if (dk != ~0u) {
      const uint32_t before = __popc(m & ((1u << lane) - 1));
      b.res[4ull * r] = cntd[dk] + before;
    }
    __syncwarp();
    if (dk != ~0u && lane == (uint32_t)(__ffs(m) - 1)) cntd[dk] += __popc(m);
    __syncwarp();
  }
}
__global__ void k_no_assign(BatchDev b, TpccParams tp) {
  extern __shared__ long long cntd[];
  no_assign_body(b, tp, blockIdx.x, cntd);
}


// ORDER.aux[row] = first ORDER_LINE row of the order if its cnt lines sit in consecutive rows
__global__ void k_build_olrow() {
  const DevTable& TOr = c_tabs[TO];
  const DevTable& TOL_ = c_tabs[TOL];
  const uint64_t n = *TOr.n_rows;
  for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < n; r += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t first = ROW_NONE;
    if (TOr.valid[r]) {
      const uint64_t okey = TOr.rowkey[r];
      const uint32_t cnt = (uint32_t)rd(TOr, O_OL_CNT, (uint32_t)r);
      first = probe(TOL_, okey * 16 + 1);
      for (uint32_t l = 1; l < cnt && first != ROW_NONE; ++l) {
        const uint64_t row = (uint64_t)first + l;
        if (row >= *TOL_.n_rows || !TOL_.valid[row] || TOL_.rowkey[row] != okey * 16 + l + 1) first = ROW_NONE;
      }
    }
    TOr.aux[r] = first;
  }
}

void tpcc_build_olrow(cudaStream_t s) {
  k_build_olrow<<<148 * 8, 256, 0, s>>>();
  note_launch();
}

// ---- host side ------------------------------------------------------------------------------------
template <class T>
static cudaError_t dm(T** p, size_t n) {
  return cudaMalloc(reinterpret_cast<void**>(p), std::max<size_t>(n, 1) * sizeof(T));
}

int tpcc_alloc(TpccDev& t, uint32_t max_txns, uint32_t nw, int* shared_by_name) {
  t.max_txns = max_txns;
  t.nw = nw;
  if (!nw) return 0;
  if (nw > 1000) return LTPG_EINVAL;
  t.dsz = nw * 10 + 11;
  // (the single-launch path counts in 32-rank chunks: up to 16384 / 32 of them)
  const uint64_t chunks = std::max<uint64_t>((max_txns + NO_CHUNK - 1) / NO_CHUNK,
                                             (std::min<uint64_t>(max_txns, 16384) + SMALL_CHUNK - 1) / SMALL_CHUNK);
  t.owns_by_name = shared_by_name == nullptr;
  if (shared_by_name) t.by_name = shared_by_name;
  else if (dm(&t.by_name, (uint64_t)t.dsz * 1000)) return LTPG_ENOMEM;
  if (dm(&t.list, (uint64_t)NTYPES * max_txns) || dm(&t.clist, (uint64_t)NTYPES * max_txns) ||
      dm(&t.log, (uint64_t)max_txns * TLOG) || dm(&t.no_pref, max_txns + 1ull) ||
      dm(&t.dk_of, max_txns) || dm(&t.chunk_cnt, chunks * t.dsz) || dm(&t.dist_base, t.dsz) || dm(&t.misc, 16) ||
      dm(&t.chunk_tot, chunks + 1) || dm(&t.dl_min, nw + 1ull))
    return LTPG_ENOMEM;
  SlScratch& sl = t.sl;
  if (dm(&sl.minr, t.dsz) || dm(&sl.slot, t.dsz) || dm(&sl.dk, t.dsz) || dm(&sl.cnt, 1) ||
      dm(&sl.low, (uint64_t)t.dsz * SL_T) || dm(&sl.nx, t.dsz) || dm(&sl.rows, (uint64_t)t.dsz * SL_SLOTS) ||
      dm(&sl.nd, t.dsz) || dm(&sl.rowd, t.dsz) || dm(&sl.m, t.dsz))
    return LTPG_ENOMEM;
  if (t.owns_by_name) cudaMemset(t.by_name, 0, (uint64_t)t.dsz * 1000 * sizeof(int));
  if (cudaStreamCreateWithFlags(&t.side, cudaStreamNonBlocking) != cudaSuccess) return LTPG_ECUDA;
  for (int k = 0; k < 2; ++k)
    if (cudaEventCreateWithFlags(&t.fork[k], cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&t.join[k], cudaEventDisableTiming) != cudaSuccess)
      return LTPG_ECUDA;
  return 0;
}

void tpcc_free(TpccDev& t) {
  if (t.side) cudaStreamDestroy(t.side);
  for (int k = 0; k < 2; ++k) {
    if (t.fork[k]) cudaEventDestroy(t.fork[k]);
    if (t.join[k]) cudaEventDestroy(t.join[k]);
  }
  if (!t.owns_by_name) t.by_name = nullptr;
  void* ps[] = {t.by_name, t.list, t.clist, t.log, t.no_pref, t.dk_of, t.chunk_cnt, t.dist_base, t.misc, t.chunk_tot,
                t.dl_min,
                t.sl.minr, t.sl.slot, t.sl.dk, t.sl.cnt, t.sl.low, t.sl.nx, t.sl.rows, t.sl.nd, t.sl.rowd, t.sl.m};
  for (void* p : ps)
    if (p) cudaFree(p);
  t = TpccDev{};
}

// Static secondary index ("primary and secondary hash tables"): (w, d, C_LAST) ->
// the customer at position ceil(n/2) when sorted by C_FIRST (TPC-C 2.5.2.2); built at load.
int tpcc_build_secondary(TpccDev& t, const uint64_t* keys, const int64_t* cols, uint64_t n, uint32_t nw) {
  if (!t.by_name || !n) return 0;
  std::map<uint64_t, std::vector<std::pair<int64_t, int64_t>>> g;
  for (uint64_t r = 0; r < n; ++r) {
    const uint64_t k = keys[r], dk = (k - 1) / 3000, c = (k - 1) % 3000 + 1;
    const int64_t last = cols[C_LAST * n + r], first = cols[C_FIRST * n + r];
    if (dk >= t.dsz || last < 0 || last > 999) continue;
    g[dk * 1000 + (uint64_t)last].push_back({first, (int64_t)c});
  }
  std::vector<int> dense((uint64_t)t.dsz * 1000, 0);
  for (auto& kv : g) {
    auto& v = kv.second;
    std::sort(v.begin(), v.end());
    dense[kv.first] = (int)v[(v.size() + 1) / 2 - 1].second;
  }
  (void)nw;
  return cudaMemcpy(t.by_name, dense.data(), dense.size() * sizeof(int), cudaMemcpyHostToDevice) == cudaSuccess
             ? 0
             : LTPG_ECUDA;
}

constexpr uint32_t AGG_DSZ_MAX = 4096;  // per-block D_YTD aggregation up to ~400 warehouses (32 KB)
static size_t wb_smem(const TpccDev& t) {
  return ((size_t)t.nw + 1 + (t.dsz <= AGG_DSZ_MAX ? t.dsz : 0)) * sizeof(long long);
}
constexpr uint32_t HOT_SMEM_MAX = 24 * 1024;  // execute's shared-memory W / D marks: up to ~190 warehouses
static uint32_t hot_words(const TpccDev& t, const BatchDev& b) {
  // off for the A/B and NEXT-3 configurations that measure the global mark path itself
  if (b.flags & (LTPG_FLAG_NO_MARK_FILTER | LTPG_FLAG_LARGE_BUCKETS)) return 0;
#ifdef LTPG_NO_HOT_MARKS
  return 0;
#endif
  const uint32_t words = t.nw + 30 * t.nw;
  return words * sizeof(mark_t) <= HOT_SMEM_MAX ? words : 0;
}
static TpccParams params_of(TpccDev& t, const BatchDev& b, bool committed_lists) {
  const uint32_t n = b.n_txns;
  return TpccParams{t.clist, committed_lists ? t.clist : t.list, committed_lists ? t.misc + M_CCOUNT : b.kcount, t.log,
                    t.no_pref, t.dk_of, t.chunk_cnt, t.dist_base, t.misc, t.by_name,
                    t.nw, t.dsz, t.max_txns, (n + NO_CHUNK - 1) / NO_CHUNK, t.chunk_tot, t.dl_min,
                    committed_lists && t.dsz <= AGG_DSZ_MAX ? t.dsz : 0u, committed_lists ? 0u : hot_words(t, b),
                    10u, false, t.dsz <= COLSCAN_TILED_DSZ};
}
static uint32_t phase_grid(uint32_t n) {
  const uint64_t warps = (uint64_t)n + NTYPES;  // upper bound (StockLevel: 1 warp/txn)
  return (uint32_t)std::min<uint64_t>((warps + 7) / 8, 148 * 16);
}
// One wave of resident blocks per phase (the grid-stride warp loop covers every slot): the
// per-block fixed costs -- the error-word barrier, execute's shared-memory mark init and flush,
// write-back's last-block counter -- are paid 148 x (blocks / SM) times per batch instead of
// once per 8 warp slots (write-back visits only the committed txns: most of a full-size grid
// had nothing to do but those fixed costs)
template <int PH>
static uint32_t resident_grid(uint32_t n, size_t smem) {
  static int per_sm[3][2] = {{0, 0}, {0, 0}, {0, 0}};  // by phase, by dynamic shared memory or not
  int& b = per_sm[PH][smem ? 1 : 0];
  if (!b && cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_tpcc_phase<PH, TM_MAIN>,
                                                          PH == PH_EXEC ? LTPG_EXEC_THREADS : 256, smem) != cudaSuccess)
    b = 2;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return std::min<uint32_t>(phase_grid(n), (uint32_t)(std::max(b, 1) * sms));
}

// cleared: misc and dl_min were reset by the batch's first kernel (k_batch_init, partition 0)
int tpcc_front(TpccDev& t, BatchDev& b, cudaStream_t s, cudaEvent_t* ev, bool cleared) {
  if (!t.nw) return LTPG_EINVAL;
  const uint32_t n = b.n_txns;
  const TpccParams tp = params_of(t, b, false);
  if (!cleared) {
    cudaMemsetAsync(t.misc, 0, 16 * sizeof(uint32_t), s);
    cudaMemsetAsync(t.dl_min, 0xFF, (t.nw + 1) * sizeof(uint32_t), s);
  }
  if (b.nparts > 1)
    k_tpcc_group<true><<<(n + 255) / 256, 256, 0, s>>>(b, tp);  // + the capacity check (last block)
  else
    k_tpcc_group4<<<(n + 1023) / 1024, 256, 0, s>>>(b, tp);  // (1 txn / thread: tpcc_c5 +2.5 us, c4 same)
  note_launch(1);
  if (ev) record_stage(ev[2], s);
  // NEXT-3: popularity from this batch's per-procedure counts -> bucket sizes
  if (t.h_tab) launch_popularity(t.h_tab, t.n_tab, b.kcount, n, t.d_su, t.popular, s);
  // StockLevel (shared per district) on a side stream, concurrently with the other procedures
  const SlScratch sl = t.sl;
  cudaEventRecord(t.fork[0], s);
  cudaStreamWaitEvent(t.side, t.fork[0], 0);
  cudaMemsetAsync(sl.minr, 0xFF, (size_t)t.dsz * sizeof(uint32_t), t.side);
  cudaMemsetAsync(sl.cnt, 0, sizeof(uint32_t), t.side);
  k_sl_claim<<<148 * 2, 256, 0, t.side>>>(b, tp, sl);
  k_sl_district<<<148 * 2, 256, 0, t.side>>>(b, sl);
  cudaEventRecord(t.join[0], t.side);
  k_tpcc_phase<PH_EXEC, TM_MAIN><<<resident_grid<PH_EXEC>(n, tp.hot_words * sizeof(mark_t)), LTPG_EXEC_THREADS,
                                   tp.hot_words * sizeof(mark_t), s>>>(b, tp);
  cudaStreamWaitEvent(s, t.join[0], 0);  // detection reads the marks of every execute warp
  note_launch(3);
  if (t.h_tab) launch_bucket_reduce(t.h_tab, t.n_tab, t.d_su, s);  // NEXT-3 large-sized buckets (if any)
  if (ev) record_stage(ev[3], s);
  cudaEventRecord(t.fork[1], s);
  cudaStreamWaitEvent(t.side, t.fork[1], 0);
  k_sl_detect<<<148 * 2, 256, 0, t.side>>>(b, sl);
  k_sl_txn<<<148 * 2, 256, 0, t.side>>>(b, tp, sl);
  cudaEventRecord(t.join[1], t.side);
  k_tpcc_phase<PH_DETECT, TM_MAIN><<<resident_grid<PH_DETECT>(n, 0), 256, 0, s>>>(b, tp);
  cudaStreamWaitEvent(s, t.join[1], 0);
  note_launch(3);
  return cudaGetLastError() == cudaSuccess ? 0 : LTPG_ECUDA;
}

int tpcc_back(TpccDev& t, BatchDev& b, uint32_t* scan_scratch, cudaStream_t s) {
  (void)scan_scratch;  // the o_id prefix scans inside k_no_chunk / k_no_colscan
  const uint32_t n = b.n_txns;
  const TpccParams tp = params_of(t, b, false);
  // committed txns re-listed per type (write-back warps only visit committed txns) -- inside
  // k_no_chunk when every txn touches this partition -- and the fetch-ADD pre-images of
  // D_NEXT_O_ID and append positions of committed NewOrders: per-chunk histograms + in-chunk
  // prefixes, column scans (+ chunk bases), assignment in rank order
  const size_t smem = (size_t)t.dsz * sizeof(uint32_t);
  if (b.nparts <= 1) {
    k_no_chunk<true><<<tp.n_chunks, 256, smem, s>>>(b, tp);
  } else {
    k_tpcc_relist<<<(n + 255) / 256, 256, 0, s>>>(b, tp);
    k_no_chunk<false><<<tp.n_chunks, 256, smem, s>>>(b, tp);
    note_launch();
  }
  if (t.dsz > COLSCAN_TILED_DSZ && !tp.cc_dm)
    k_no_colscan_tiled<<<(t.dsz + 7) / 8 + 1, 256, 0, s>>>(b, tp);
  else
    k_no_colscan<<<(t.dsz + 7) / 8 + 1, 256, 0, s>>>(b, tp);
  if (2 * smem > 48 * 1024) {  // (n_warehouses <= 1000: at most 80 KB)
    static size_t set = 0;
    if (set < 2 * smem && cudaFuncSetAttribute(k_no_assign, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                               (int)(2 * smem)) == cudaSuccess)
      set = 2 * smem;
  }
  k_no_assign<<<tp.n_chunks, 32, 2 * smem, s>>>(b, tp);
  note_launch(3);
  k_tpcc_phase<PH_WB, TM_MAIN><<<resident_grid<PH_WB>(n, wb_smem(t)), 256, wb_smem(t), s>>>(b, params_of(t, b, true));  // + row counters
  note_launch(1);
  return cudaGetLastError() == cudaSuccess ? 0 : LTPG_ECUDA;
}


// ---- small batches: a1..a8 in ONE cooperative launch ---------------------------------------
// A single-partition batch of <= 16384 txns (BASELINE configs[1]: 1 warehouse, 16k NewOrder /
// Payment) runs each stage in a few microseconds, so the ~14 kernel boundaries of the multi-kernel
// path (and the StockLevel side-stream joins) were most of its latency.  Here the same stage
// bodies run in one co-resident grid separated by grid-wide barriers:
//   S1 a1/a2 validation + per-type lists (+ the StockLevel district claims, the batch's clears)
//   S2 a4/a5 execute + marks; StockLevel districts          S3 a6 detection; StockLevel M
//   S4 StockLevel verdicts; committed re-lists + o_id counts per 32-rank chunk
//   S5 o_id column scans + chunk bases   (the a8 block: commit bitmask, counts, abort list)
//   S6 a7 write-back, each committed NewOrder's o_id = district base + chunk prefix + in-chunk rank
// then the last block to finish advances the append-row counters, publishes the slot's result
// words into mapped host memory and returns the batch scratch to its rest state (misc counters,
// Delivery minima, StockLevel claims, the slot's small words: the next single-launch batch needs
// no clearing pass; capi.cu clears them once after a multi-kernel batch).  Same device code as
// the multi-kernel path (the bodies above), hence result-identical.  Work stages run on blocks
// [0, G-1); block G-1 only computes a8 (it leaves the barrier protocol after S4).
__global__ void __launch_bounds__(256, 2) k_tpcc_small(BatchDev b, TpccParams tx, TpccParams tw, SlScratch sl,
                                                       SmallOut o) {
  TSM_PASS(0);
  uint32_t* bar = o.bar;  // zero at launch, cleared at the end
  const uint32_t G = gridDim.x, W = G - 1;
  const bool fin = blockIdx.x == G - 1;
  const uint32_t n = b.n_txns;
  // S1: the batch's clears for the later stages (append reservations, batch scalars -- read with
  // ld.global.nc by b_epoch after the barrier, no SM cached their line before -- user-abort flags)
  if (blockIdx.x == 0) {
    if (threadIdx.x < MAXT) o.reserve[threadIdx.x] = 0;
    if (threadIdx.x == 0) {
      o.vars->epoch = o.host ? o.host->epoch : o.epoch;
      o.vars->clock = o.host ? o.host->clock : o.clock;
    }
  }
  if (!fin) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += W * blockDim.x) b.ua[i] = 0;
    for (uint32_t vb = blockIdx.x; vb < (n + blockDim.x - 1) / blockDim.x; vb += W)
      tpcc_group_body<false, true>(b, tx, vb, sl);
  }
  TSM_WORK(1);
  grid_barrier_to(bar, G);
  TSM_PASS(1);
  if (!fin) {  // S2
    tpcc_phase_body<PH_EXEC, TM_MAIN, true>(b, tx, blockIdx.x, W);
    sl_district_body(b, sl, blockIdx.x, W);
  }
  TSM_WORK(2);
  grid_barrier_to(bar, 2 * G);
  TSM_PASS(2);
  if (!fin) {  // S3
    tpcc_phase_body<PH_DETECT, TM_MAIN, true>(b, tx, blockIdx.x, W);
    sl_detect_body(b, sl, blockIdx.x, W);
  }
  TSM_WORK(3);
  grid_barrier_to(bar, 3 * G);
  TSM_PASS(3);
  if (!fin) {  // S4
    sl_txn_body(b, tx, sl, blockIdx.x, W);
    for (uint32_t vb = blockIdx.x; vb < (n + blockDim.x - 1) / blockDim.x; vb += W) no_chunk32_body(b, tx, vb);
  } else {  // every district's snapshot D_NEXT_O_ID (the o_id bases; S5 then only adds)
    const DevTable& TDi = c_tabs[TD];
    const uint32_t dmask = *b.dense_live;
    for (uint32_t dk = 11 + threadIdx.x; dk < tx.dsz; dk += blockDim.x) {  // kD(1, 1) = 11
      const uint32_t row_d = rowof(TDi, TD, dk, dmask);
      if (row_d != ROW_NONE) tx.dist_base[dk] = rd(TDi, D_NEXT_O_ID, row_d);
    }
  }
  TSM_WORK(4);
  grid_barrier_to(bar, 4 * G);  // every verdict is final
  TSM_PASS(4);
  const bool ok = *(volatile uint32_t*)b.err == 0;  // uniform: raised before the last barrier
  if (fin) {  // a8
    if (ok) finalize_block(n, o, [&](uint32_t r) { return b.status[r]; });
    else if (threadIdx.x < 17 && (threadIdx.x || o.write0)) o.dsmall[threadIdx.x] = 0;  // failed batch: no counts
    TSM_WORK(8);
  } else {
    const uint32_t ncs = (tx.dsz + 7) / 8 + 1;  // S5
    if (ok)
      for (uint32_t vb = blockIdx.x; vb < ncs; vb += W) no_colscan_body<true>(b, tx, vb, ncs);
    TSM_WORK(5);
    grid_barrier_to(bar, 4 * G + W);
    TSM_PASS(5);
    TSM_PASS(6);
    tpcc_phase_body<PH_WB, TM_MAIN, true>(b, tw, blockIdx.x, W);  // S6 (o_ids computed inline)
    TSM_WORK(7);
  }
  __shared__ bool last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd(b.done, 1u) == G - 1;
  }
  __syncthreads();
  if (!last) return;
  __threadfence();
  if (threadIdx.x == 0) tpcc_advance_tail(b, tw);  // (nothing when the batch failed)
  if (threadIdx.x < 17)
    o.host_small[threadIdx.x] = reinterpret_cast<volatile uint32_t*>(o.dsmall)[threadIdx.x] |
                                (threadIdx.x == 0 ? *reinterpret_cast<volatile uint32_t*>(b.err) : 0u);
  const uint32_t nsl = *(volatile uint32_t*)sl.cnt;
  for (uint32_t i = threadIdx.x; i < nsl; i += blockDim.x) sl.minr[sl.dk[i]] = 0xFFFFFFFFu;
  for (uint32_t w = threadIdx.x; w <= tx.nw; w += blockDim.x) tx.dl_min[w] = ~0u;
  __syncthreads();
  if (threadIdx.x < 16) {
    b.err[threadIdx.x] = 0;  // err .. done
    tx.misc[threadIdx.x] = 0;
  }
  if (threadIdx.x == 0) *bar = 0;
  if (threadIdx.x == 0) *sl.cnt = 0;
#ifdef LTPG_SMALL_TS
  if (threadIdx.x == 0) {
    unsigned long long t_;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));
    volatile unsigned long long* p = g_tsm[0];
    volatile unsigned long long* w = g_tsm[1];
    printf("k_tpcc_small n=%u G=%u ns from start: pass B1 %lld B2 %lld B3 %lld B4 %lld B5 %lld B6 %lld end %lld | "
           "work end S1 %lld S2 %lld S3 %lld S4 %lld S5 %lld S5-districts %lld S7 %lld a8 %lld S5-chunks %lld\n", n, G,
           (long long)(p[1] - p[0]), (long long)(p[2] - p[0]), (long long)(p[3] - p[0]), (long long)(p[4] - p[0]),
           (long long)(p[5] - p[0]), (long long)(p[6] - p[0]), (long long)(t_ - p[0]), (long long)(w[1] - p[0]),
           (long long)(w[2] - p[0]), (long long)(w[3] - p[0]), (long long)(w[4] - p[0]), (long long)(w[5] - p[0]),
           (long long)(w[6] - p[0]), (long long)(w[7] - p[0]), (long long)(w[8] - p[0]), (long long)(w[9] - p[0]));
    for (int k = 0; k < 10; ++k) w[k] = 0;
  }
#endif
}

uint32_t tpcc_small_max_txns() { return 16384; }
bool tpcc_small_fits(const TpccDev& t) { return t.nw >= 1 && t.nw <= TPCC_SMALL_MAX_W; }

void tpcc_small_clear(TpccDev& t, cudaStream_t s) {
  cudaMemsetAsync(t.misc, 0, 16 * sizeof(uint32_t), s);
  cudaMemsetAsync(t.dl_min, 0xFF, (t.nw + 1) * sizeof(uint32_t), s);
  cudaMemsetAsync(t.sl.minr, 0xFF, (size_t)t.dsz * sizeof(uint32_t), s);
  cudaMemsetAsync(t.sl.cnt, 0, sizeof(uint32_t), s);
}

int launch_tpcc_small(TpccDev& t, const BatchDev& b, const SmallOut& o, cudaStream_t s) {
  TpccParams tx = params_of(t, b, false), tw = params_of(t, b, true);
  tx.n_chunks = tw.n_chunks = (b.n_txns + SMALL_CHUNK - 1) / SMALL_CHUNK;
  tx.chunk_shift = tw.chunk_shift = 5;
  static_assert(SMALL_CHUNK == 32, "one warp per chunk");
  tw.oid_inline = true;
  tx.cc_dm = tw.cc_dm = true;  // (<= 64 warehouses)
  const size_t smem = std::max((size_t)tx.hot_words * sizeof(mark_t), wb_smem(t));  // execute's hm / write-back's agg
  static int ps = 0, sms = 0;  // co-resident blocks per SM at the last dynamic shared memory size
  static size_t ps_smem = ~(size_t)0;
  if (smem != ps_smem) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ps, k_tpcc_small, 256, smem) != cudaSuccess || ps < 1) ps = 1;
    ps_smem = smem;
  }
  // about 8 txns per warp (execute's NewOrder slots) + the a8 block; co-resident
  const uint32_t want = (b.n_txns + 63) / 64 + 1;
  const uint32_t grid = std::max<uint32_t>(2, std::min<uint32_t>(want, (uint32_t)(ps * sms)));
  BatchDev bb = b;
  TpccParams a = tx, c = tw;
  SlScratch sl = t.sl;
  SmallOut so = o;
  void* args[] = {&bb, &a, &c, &sl, &so};
  cudaLaunchCooperativeKernel((const void*)k_tpcc_small, dim3(grid), dim3(256), args, smem, s);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : LTPG_ECUDA;
}

}  // namespace ltpg
