// OPS-mode kernels (YCSB and generic key/value transactions).
//
//  K-group   validate the batch (a1) and decompose it into per-kind op lists so
//            every execute warp runs one op kind (adaptive warp division)
//  K-claim   INSERT keys claim their index slot with a provisional row (a3)
//  K-exec    readMem / recordLS / recordTID: snapshot reads, result
//            slots, epoch-tagged atomicMin marks per conflict unit (a4, a5)
//  K-detect  rcheck / wcheck: per-txn OR of the RAW/WAW test (a6)
//  K-wb      getStatus -> writeMem: committed write sets only (a7)
#include <cooperative_groups.h>

#include <algorithm>
#include <cstdio>

#include "ltpg_internal.cuh"
#include "small.cuh"

namespace cg = cooperative_groups;

namespace ltpg {

LTPG_DEFINE_TABLE_UPLOAD(upload_tables_ops)

constexpr int OPS_MAX_TXN_OPS = 256;

__device__ __forceinline__ ltpg_op load_op(const ltpg_op* ops, uint32_t i) {
  const ulonglong2 v = *reinterpret_cast<const ulonglong2*>(ops + i);
  ltpg_op o;
  o.key = v.x;
  o.kind = (uint8_t)(v.y);
  o.table = (uint8_t)(v.y >> 8);
  o.col = (uint16_t)(v.y >> 16);
  o.aux = (uint32_t)(v.y >> 32);
  return o;
}

__device__ __forceinline__ bool op_valid(uint32_t n_tables, const ltpg_op& o) {
  if (o.table >= n_tables) return false;
  const DevTable& T = c_tabs[o.table];
  if (!T.defined || !T.has_pk || o.kind > LTPG_SCAN || o.key == KEY_EMPTY) return false;
  switch (o.kind) {
    case LTPG_SELECT: return o.col < T.n_cols;
    case LTPG_UPDATE: return o.col < T.n_cols && col_group(T, o.col) != LTPG_STATIC && !col_is_add(T, o.col);
    case LTPG_ADD: return o.col < T.n_cols && col_is_add(T, o.col);
    case LTPG_INSERT: return T.n_groups > 0;
    case LTPG_DELETE: return T.n_groups > 0 && !T.has_static;
    default:  // SCAN
      if (o.col != LTPG_COL_COUNT && o.col >= T.n_cols) return false;
      return o.aux == 0 || o.key <= KEY_EMPTY - o.aux;
  }
}

__device__ __forceinline__ bool is_write_kind(uint8_t k) {
  return k == LTPG_UPDATE || k == LTPG_ADD || k == LTPG_INSERT || k == LTPG_DELETE;
}

// Does this partition handle (part of) op o?  Key ranges are contiguous, so a SCAN touches
// the partitions between the owners of its first and last key.
__device__ __forceinline__ bool op_touches(const BatchDev& b, const ltpg_op& o) {
  if (b.nparts <= 1) return true;
  const DevTable& T = c_tabs[o.table];
  if (T.owner_rule != 2) return b.part == 0;
  const uint32_t p0 = part_of_key(2, o.key, b.key_space, b.nparts);
  if (o.kind != LTPG_SCAN || o.aux <= 1) return p0 == b.part;
  const uint32_t p1 = part_of_key(2, o.key + o.aux - 1, b.key_space, b.nparts);
  return p0 <= b.part && b.part <= p1;
}

// ---- a1: validation of one txn (R2-R4, R10) over a staged or global op accessor --------
template <class Get>
__device__ __forceinline__ bool validate_txn(uint32_t n_tables, const BatchDev& b, uint32_t r, bool staged,
                                             uint32_t w0, uint32_t w1, Get get, uint32_t& b0, uint32_t& b1,
                                             uint64_t& cnt64, uint32_t& ins_tables, uint32_t& insdel) {
  bool bad = false;
  if (r > 0 && b.tid[r] <= b.tid[r - 1]) bad = true;  // TIDs strictly increasing
  b0 = b.op_begin[r];
  b1 = b.op_begin[r + 1];
  if (r == 0 && b0 != 0) bad = true;
  if (r == b.n_txns - 1 && b1 != b.n_ops) bad = true;
  if (b1 < b0 || b1 > b.n_ops || b1 - b0 > OPS_MAX_TXN_OPS || (staged && (b0 < w0 || b1 > w1))) {
    bad = true;
    b1 = b0;
  }
  for (uint32_t i = b0; i < b1; ++i) {
    const ltpg_op o = get(i);
    if (o.kind == LTPG_INSERT || o.kind == LTPG_DELETE) insdel |= 1u << (o.table & 31);
    if (!op_valid(n_tables, o)) { bad = true; continue; }
    if (!op_touches(b, o)) continue;
    cnt64 += 1ull << (10 * o.kind);
    if (o.kind == LTPG_INSERT) ins_tables |= 1u << o.table;
  }
  // R10: a written key is touched by no other op of the txn (no read-your-writes)
  for (uint32_t i = b0 + 1; i < b1 && !bad; ++i) {
    const ltpg_op a = get(i);
    const uint64_t alo = a.key, ahi = a.kind == LTPG_SCAN ? a.key + a.aux : a.key + 1;
    for (uint32_t j = b0; j < i; ++j) {
      const ltpg_op c = get(j);
      if (c.table != a.table) continue;
      const uint64_t clo = c.key, chi = c.kind == LTPG_SCAN ? c.key + c.aux : c.key + 1;
      if (!(alo < chi && clo < ahi)) continue;
      if (is_write_kind(a.kind) || is_write_kind(c.kind) || (a.kind != LTPG_SCAN && c.kind != LTPG_SCAN)) {
        bad = true;
        break;
      }
    }
  }
  return bad;
}

__device__ __forceinline__ ltpg_op unpack_op(ulonglong2 v) {
  ltpg_op o;
  o.key = v.x;
  o.kind = (uint8_t)(v.y);
  o.table = (uint8_t)(v.y >> 8);
  o.col = (uint16_t)(v.y >> 16);
  o.aux = (uint32_t)(v.y >> 32);
  return o;
}

// ---- K-group: validation + decomposition into per-kind lists (one thread per txn) ----
constexpr uint32_t GROUP_STAGE = 352;  // ops per warp staged in shared memory (YCSB: 32 x 10 = 320)
template <bool GROUPED>
__device__ __forceinline__ void ops_validate_group_body(uint32_t n_tables, const BatchDev& b,
                                                        ltpg_op (*stage)[GROUP_STAGE]) {
  constexpr uint32_t STAGE = GROUP_STAGE;
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r < b.n_txns) {  // validation's scalar loads, in flight while the op records are staged
    asm volatile("prefetch.global.L1 [%0];" ::"l"(b.tid + r));
    asm volatile("prefetch.global.L1 [%0];" ::"l"(b.op_begin + r));
  }
  const int lane = threadIdx.x & 31;
  const uint32_t wib = threadIdx.x >> 5;
  bool bad = false;
  uint32_t b0 = 0, b1 = 0;
  uint64_t cnt64 = 0;  // per-kind op counts, 10 bits each (no dynamically indexed arrays)
  uint32_t my_ins_tables = 0, my_insdel = 0;
  // the warp's ops form one contiguous range: stage it with coalesced 16-byte loads
  const uint32_t r0 = r - lane;
  const uint32_t rl = min(r0 + 32, b.n_txns);
  uint32_t w0 = 0, w1 = 0;
  if (r0 < b.n_txns) {
    w0 = b.op_begin[r0];
    w1 = b.op_begin[rl];
  }
  const bool staged = r0 < b.n_txns && w1 >= w0 && w1 - w0 <= STAGE && w1 <= b.n_ops;
  if (staged)
    for (uint32_t q = w0 + lane; q < w1; q += 32)
      *reinterpret_cast<ulonglong2*>(&stage[wib][q - w0]) = *reinterpret_cast<const ulonglong2*>(b.ops + q);
  __syncwarp();
  auto get = [&](uint32_t q) -> ltpg_op {
    if (staged) return unpack_op(*reinterpret_cast<const ulonglong2*>(&stage[wib][q - w0]));
    return load_op(b.ops, q);
  };
  if (r < b.n_txns) {
    bad = validate_txn(n_tables, b, r, staged, w0, w1, get, b0, b1, cnt64, my_ins_tables, my_insdel);
    b.txn_ins[r] = (uint32_t)(cnt64 >> (10 * LTPG_INSERT)) & 1023u;
    if (bad) atomicOr(b.err, ERR_EINVAL);
  }
  my_ins_tables = __reduce_or_sync(0xffffffffu, my_ins_tables);
  if (lane == 0 && my_ins_tables) atomicOr(b.ins_tables, my_ins_tables);
  my_insdel = __reduce_or_sync(0xffffffffu, my_insdel);
  if (lane == 0 && my_insdel) atomicOr(b.insdel, my_insdel);
  if (!GROUPED) {
    // one flat list in op order (region 0); INSERTs are still listed for K-claim
    if (r < b.n_txns)
      for (uint32_t i = b0; i < b1; ++i) b.items[i] = (unsigned long long)i | ((unsigned long long)r << 32);
    if (r == 0) b.kcount[0] = b.n_ops;
    if (r < b.n_txns && !bad)
      for (uint32_t i = b0; i < b1; ++i)
        if (b.ops[i].kind == LTPG_INSERT && op_touches(b, load_op(b.ops, i))) {
          uint32_t p = atomicAdd(b.kcount + LTPG_INSERT, 1u);
          b.items[(uint64_t)LTPG_INSERT * b.max_ops + p] = (unsigned long long)i | ((unsigned long long)r << 32);
        }
    return;
  }
  // block-aggregated reservation in the per-kind lists: one atomicAdd per block and kind
  uint32_t ck[NKINDS], pos[NKINDS];
#pragma unroll
  for (int k = 0; k < NKINDS; ++k) ck[k] = (uint32_t)(cnt64 >> (10 * k)) & 1023u;
  block_reserve<NKINDS>(ck, b.kcount, pos);
  if (r < b.n_txns && !bad)
    for (uint32_t i = b0; i < b1; ++i) {
      const ltpg_op o = get(i);
      if (!op_touches(b, o)) continue;
      const uint8_t k = o.kind;
      uint32_t p = 0;
#pragma unroll
      for (int kk = 0; kk < NKINDS; ++kk)
        if (kk == k) p = pos[kk]++;
      b.items[(uint64_t)k * b.max_ops + p] = (unsigned long long)i | ((unsigned long long)r << 32);
    }
}
template <bool GROUPED>
__global__ void __launch_bounds__(256) k_ops_validate_group(uint32_t n_tables, BatchDev b) {
  __shared__ __align__(16) ltpg_op stage[8][GROUP_STAGE];
  ops_validate_group_body<GROUPED>(n_tables, b, stage);
}

void launch_ops_validate_group(uint32_t n_tables, const BatchDev& b, bool grouped,
                               cudaStream_t s) {
  uint32_t blocks = (b.n_txns + 255) / 256;
  if (grouped)
    k_ops_validate_group<true><<<blocks, 256, 0, s>>>(n_tables, b);
  else
    k_ops_validate_group<false><<<blocks, 256, 0, s>>>(n_tables, b);
  note_launch();
}

// ---- K-claim: INSERT keys claim their slot; provisional row = n_rows + rank of the
//      insert in (rank, op) order; atomicMin makes the earliest inserter own the unit ----
__device__ __forceinline__ void ops_claim_body(const BatchDev& b) {
  if (*b.err) return;
  const uint32_t n = b.kcount[LTPG_INSERT];
  const unsigned long long* list = b.items + (uint64_t)LTPG_INSERT * b.max_ops;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    unsigned long long it = list[i];
    uint32_t oi = (uint32_t)it, r = (uint32_t)(it >> 32);
    ltpg_op o = load_op(b.ops, oi);
    const DevTable& T = c_tabs[o.table];
    uint32_t j = 0;
    for (uint32_t q = b.op_begin[r]; q < oi; ++q)
      j += b.ops[q].kind == LTPG_INSERT && op_touches(b, load_op(b.ops, q));
    uint32_t prov = (uint32_t)(*T.n_rows + b.base[o.table] + b.txn_ins[r] + j);
    IdxSlot* sl = idx_find_or_insert(T, o.key);
    if (!sl) { atomicOr(b.err, ERR_EINTERNAL); continue; }
    if (*reinterpret_cast<volatile unsigned*>(&sl->row) != ROW_NONE) continue;  // present in S
    atomicMin(&sl->claim, prov);
  }
}
__global__ void __launch_bounds__(256) k_ops_claim(BatchDev b) { ops_claim_body(b); }

void launch_ops_claim(const BatchDev& b, cudaStream_t s) {
  k_ops_claim<<<148 * 4, 256, 0, s>>>(b);
  note_launch();
}

// ---- K-exec ---------------------------------------------------------------------------
__device__ __forceinline__ void mark_read(const DevTable& T, uint32_t g, uint32_t row, mark_t tag,
                                          bool filter) {
  if (T.rmarks) mark_unit(T, MK_R, g, row, tag, filter);  // NEXT-1 only: min reader rank
}

// uref bit 58: absent key read before K-claim ran (fused path); K-detect probes it for a claim
constexpr uint64_t UREF_RECHECK = 1ull << 58;

__device__ __forceinline__ void exec_one(const BatchDev& b, uint32_t oi, uint32_t r, const ltpg_op& o,
                                         bool filter, uint32_t dmask, bool pre_claim = false) {
  const DevTable& T = c_tabs[o.table];
  const mark_t tag = epoch_tag(b_epoch(b)) | r;
  uint32_t row, claim;
  long long res = LTPG_NOT_FOUND;
  uint64_t uref = 0;
  if (!op_touches(b, o)) return;  // another partition's op (flat-list mode)
  if (o.kind == LTPG_SCAN) {  // range of predefined keys; checked again in detect
    long long cnt = 0;
    unsigned long long sum = 0;
    const uint32_t gs = (o.col != LTPG_COL_COUNT && col_group(T, o.col) != LTPG_STATIC) ? col_group(T, o.col) : 0;
    for (uint64_t k = o.key; k < o.key + o.aux; ++k) {
      if (!owns_key(b, T, k)) continue;  // partitioned: this partition's part of the range
      lookup(T, o.table, dmask, k, row, claim);
      if (row != ROW_NONE) {
        ++cnt;
        if (o.col != LTPG_COL_COUNT) sum += (unsigned long long)*col_ptr_ops(T, o.col, row);
        if (T.n_groups) mark_read(T, gs, row, tag, filter);
      } else if (claim != ROW_NONE) {
        mark_read(T, 0, claim, tag, filter);
      }
    }
    b.res[oi] = o.col == LTPG_COL_COUNT ? cnt : (long long)sum;
    b.uref[oi] = make_uref(CHK_SCAN, false, false, o.table, 0, 0);
    return;
  }
  lookup(T, o.table, dmask, o.key, row, claim);
  const bool present = row != ROW_NONE;
  if (!present && o.kind != LTPG_INSERT) {
    // absent key: a READ of its existence; only an inserter of this batch can conflict
    if (claim != ROW_NONE) mark_read(T, 0, claim, tag, filter);
    uref = claim != ROW_NONE ? make_uref(CHK_RW, false, false, o.table, 0, claim)
           : pre_claim       ? (make_uref(CHK_RW, false, false, o.table, 0, 0) | UREF_RECHECK)
                             : make_uref(CHK_NONE, false, false, o.table, 0, 0);
    b.res[oi] = LTPG_NOT_FOUND;
    b.uref[oi] = uref;
    return;
  }
  switch (o.kind) {
    case LTPG_SELECT: {
      res = *col_ptr_ops(T, o.col, row);
      uint32_t g = col_group(T, o.col);
      if (g != LTPG_STATIC) mark_read(T, g, row, tag, filter);
      uref = g == LTPG_STATIC ? make_uref(CHK_NONE, false, true, o.table, 0, row)
                              : make_uref(CHK_RW, false, true, o.table, g, row);
      break;
    }
    case LTPG_UPDATE: {
      uint32_t g = col_group(T, o.col);
      res = *col_ptr_ops(T, o.col, row);  // pre-image; new value = res + arg at write-back
      mark_unit(T, MK_W, g, row, tag, filter);
      uref = make_uref(CHK_RW, false, true, o.table, g, row, true);
      break;
    }
    case LTPG_ADD: {
      uint32_t g = col_group(T, o.col);
      res = 0;
      mark_unit(T, MK_A, g, row, tag, filter);
      uref = make_uref(CHK_A, false, true, o.table, g, row, true);
      break;
    }
    case LTPG_INSERT:
      if (present) {  // duplicate key: user abort; a READ of the row
        res = 0;
        b.ua[r] = 1;
        mark_read(T, 0, row, tag, filter);
        uref = make_uref(CHK_RW, false, true, o.table, 0, row);
      } else {
        if (claim == ROW_NONE) {  // every absent INSERT key was claimed by K-claim
          atomicOr(b.err, ERR_EINTERNAL);
          return;
        }
        res = 1;
        for (uint32_t g = 0; g < T.n_groups; ++g) mark_unit(T, MK_W, g, claim, tag, filter);
        uref = make_uref(CHK_RW, true, false, o.table, 0, claim, true);
      }
      break;
    case LTPG_DELETE:
      res = 1;
      for (uint32_t g = 0; g < T.n_groups; ++g) mark_unit(T, MK_W, g, row, tag, filter);
      uref = make_uref(CHK_RW, true, true, o.table, 0, row, true);
      break;
  }
  b.res[oi] = res;
  b.uref[oi] = uref;
}

template <bool GROUPED>
__device__ __forceinline__ void ops_exec_body(const BatchDev& b, bool filter) {
  if (*b.err) return;
  const uint32_t dmask = *b.dense_live & ~*b.insdel;
  const int lane = threadIdx.x & 31;
  uint32_t cnt[NKINDS], pref[NKINDS + 1];  // fully unrolled below: registers only
  pref[0] = 0;
#pragma unroll
  for (int k = 0; k < NKINDS; ++k) {
    cnt[k] = GROUPED ? b.kcount[k] : (k == 0 ? b.n_ops : 0);
    pref[k + 1] = pref[k] + ((cnt[k] + 31) & ~31u);  // each kind padded to whole warps
  }
  const uint32_t nwarps = gridDim.x * (blockDim.x >> 5);
  for (uint32_t w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); (uint64_t)w * 32 < pref[NKINDS];
       w += nwarps) {
    const uint32_t p = w * 32;
    uint32_t k = 0, pk = 0, ck = cnt[0];
#pragma unroll
    for (int kk = 1; kk < NKINDS; ++kk)
      if (p >= pref[kk]) { k = kk; pk = pref[kk]; ck = cnt[kk]; }  // warp-uniform op kind
    const uint32_t idx = p - pk + lane;
    if (idx >= ck) continue;
    const unsigned long long it = b.items[(uint64_t)k * b.max_ops + idx];
    const uint32_t oi = (uint32_t)it, r = (uint32_t)(it >> 32);
    const ltpg_op o = load_op(b.ops, oi);
    exec_one(b, oi, r, o, filter, dmask);
  }
}
template <bool GROUPED>
__global__ void __launch_bounds__(256) k_ops_exec(BatchDev b, bool filter) { ops_exec_body<GROUPED>(b, filter); }

// ---- K-fused: a1 + warp-local kind division + a4/a5 in one pass ------------
// Each warp validates its 32 txns from shared memory, orders its own ops by kind and runs
// them 32 at a time, so a warp executes one op kind except at the few kind boundaries --
// the warp-division effect without the global lists' round trip through HBM.  INSERTs go
// to the INSERT list (K-claim, then K-exec on that list); reads of keys absent from the
// index carry UREF_RECHECK so K-detect finds claims made after this kernel.
constexpr uint32_t FUSED_STAGE = 320;  // YCSB: 32 txns x 10 ops; larger warps run unstaged
__device__ __forceinline__ void ops_fused_body(uint32_t n_tables, const BatchDev& b, bool filter,
                                               ltpg_op (*stage)[FUSED_STAGE], uint16_t (*perm)[FUSED_STAGE]) {
  constexpr uint32_t STAGE = FUSED_STAGE;
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t wib = threadIdx.x >> 5;
  const uint32_t dmask = *b.dense_live;  // INSERT/DELETE take effect at write-back only
  bool bad = false;
  uint32_t b0 = 0, b1 = 0;
  uint64_t cnt64 = 0;
  uint32_t my_ins_tables = 0, my_insdel = 0;
  const uint32_t r0 = r - lane;
  const uint32_t rl = min(r0 + 32, b.n_txns);
  uint32_t w0 = 0, w1 = 0;
  if (r0 < b.n_txns) {
    w0 = b.op_begin[r0];
    w1 = b.op_begin[rl];
  }
  const bool staged = r0 < b.n_txns && w1 >= w0 && w1 - w0 <= STAGE && w1 <= b.n_ops;
  if (staged)
    for (uint32_t q = w0 + lane; q < w1; q += 32)
      *reinterpret_cast<ulonglong2*>(&stage[wib][q - w0]) = *reinterpret_cast<const ulonglong2*>(b.ops + q);
  __syncwarp();
  auto get = [&](uint32_t q) -> ltpg_op {
    if (staged) return unpack_op(*reinterpret_cast<const ulonglong2*>(&stage[wib][q - w0]));
    return load_op(b.ops, q);
  };
  if (r < b.n_txns) {
    bad = validate_txn(n_tables, b, r, staged, w0, w1, get, b0, b1, cnt64, my_ins_tables, my_insdel);
    b.txn_ins[r] = (uint32_t)(cnt64 >> (10 * LTPG_INSERT)) & 1023u;
    if (bad) atomicOr(b.err, ERR_EINVAL);
  }
  my_ins_tables = __reduce_or_sync(0xffffffffu, my_ins_tables);
  if (lane == 0 && my_ins_tables) atomicOr(b.ins_tables, my_ins_tables);
  my_insdel = __reduce_or_sync(0xffffffffu, my_insdel);
  if (lane == 0 && my_insdel) atomicOr(b.insdel, my_insdel);
  if (bad) cnt64 = 0, b1 = b0;  // the batch fails; run nothing of this txn
  // INSERT list: warp-aggregated reservation
  const uint32_t nins = (uint32_t)(cnt64 >> (10 * LTPG_INSERT)) & 1023u;
  uint32_t ins_pos = nins;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, ins_pos, o);
    if (lane >= (uint32_t)o) ins_pos += y;
  }
  uint32_t ins_base = 0;
  if (lane == 31 && ins_pos) ins_base = atomicAdd(b.kcount + LTPG_INSERT, ins_pos);
  ins_pos += __shfl_sync(0xffffffffu, ins_base, 31) - nins;
  unsigned long long* ins_list = b.items + (uint64_t)LTPG_INSERT * b.max_ops;
  if (!staged) {  // large txns: each lane runs its own ops in op order
    for (uint32_t i = b0; i < b1; ++i) {
      const ltpg_op o = load_op(b.ops, i);
      if (!op_touches(b, o)) continue;
      if (o.kind == LTPG_INSERT) ins_list[ins_pos++] = (unsigned long long)i | ((unsigned long long)r << 32);
      else exec_one(b, i, r, o, filter, dmask, true);
    }
    return;
  }
  // warp-local kind order: inclusive scan of the packed counts (each warp total <= STAGE < 1024)
  const uint64_t mine = cnt64 & ~(1023ull << (10 * LTPG_INSERT));
  uint64_t inc = mine;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= (uint32_t)o) inc += y;
  }
  const uint64_t tot = __shfl_sync(0xffffffffu, inc, 31);
  const uint64_t excl = inc - mine;
  uint32_t pos[NKINDS], run = 0;
#pragma unroll
  for (int k = 0; k < NKINDS; ++k) {
    pos[k] = run + ((uint32_t)(excl >> (10 * k)) & 1023u);
    run += (uint32_t)(tot >> (10 * k)) & 1023u;
  }
  for (uint32_t i = b0; i < b1; ++i) {
    const ltpg_op o = get(i);
    if (!op_touches(b, o)) continue;
    if (o.kind == LTPG_INSERT) {
      ins_list[ins_pos++] = (unsigned long long)i | ((unsigned long long)r << 32);
      continue;
    }
    uint32_t p = 0;
#pragma unroll
    for (int k = 0; k < NKINDS; ++k)
      if (k == o.kind) p = pos[k]++;
    perm[wib][p] = (uint16_t)((i - w0) | (lane << 9));
  }
  __syncwarp();
  for (uint32_t q = lane; q < run; q += 32) {
    const uint32_t e = perm[wib][q];
    const uint32_t li = e & 511u;
    const ltpg_op o = unpack_op(*reinterpret_cast<const ulonglong2*>(&stage[wib][li]));
    exec_one(b, w0 + li, r0 + (e >> 9), o, filter, dmask, true);
  }
}
__global__ void __launch_bounds__(256) k_ops_fused(uint32_t n_tables, BatchDev b, bool filter) {
  __shared__ __align__(16) ltpg_op stage[8][FUSED_STAGE];
  __shared__ uint16_t perm[8][FUSED_STAGE];  // staged op index | lane << 9, ordered by kind
  ops_fused_body(n_tables, b, filter, stage, perm);
}

void launch_ops_fused(uint32_t n_tables, const BatchDev& b, bool filter, cudaStream_t s) {
  k_ops_fused<<<(b.n_txns + 255) / 256, 256, 0, s>>>(n_tables, b, filter);
  note_launch();
}

void launch_ops_exec_inserts(const BatchDev& b, bool filter, cudaStream_t s) {
  k_ops_exec<true><<<148 * 2, 256, 0, s>>>(b, filter);  // only the INSERT list is populated
  note_launch();
}

// The fused front end's INSERT tail in ONE cooperative launch (grid-wide barriers between the
// steps): exclusive scan of the per-txn insert counts -> capacity check and the partition's row
// base -> index claims -> execution of the INSERT list.  A batch without INSERTs (YCSB A/B/C, the
// common case) leaves after one load of the insert-table mask -- instead of the six dependent
// launches (3-kernel scan, capacity, claim, exec) it paid before.
// run_exec = false: ends after the claims' grid barrier (when there are INSERTs) -- the caller
// executes every kind list itself
__device__ __forceinline__ void ops_insert_tail_body(uint32_t n_tables, const BatchDev& b, bool filter,
                                                     uint32_t* partials, cg::grid_group& grid, bool run_exec = true) {
  const uint32_t n = b.n_txns;
  if (*(volatile uint32_t*)b.ins_tables == 0) {  // uniform: written by the previous kernel
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      b.txn_ins[n] = 0;
      for (uint32_t t = 0; t < n_tables; ++t) b.base[t] = b.reserve[t];  // (k_capacity with no inserts)
    }
    return;
  }
  // exclusive scan of txn_ins[0, n) in place, total in txn_ins[n]: block chunks, their sums, offsets
  __shared__ uint32_t wsum[8];
  __shared__ uint32_t carry;
  const uint32_t per = (n + gridDim.x - 1) / gridDim.x, lo = min(n, blockIdx.x * per), hi = min(n, lo + per);
  uint32_t part = 0;
  for (uint32_t i = lo + threadIdx.x; i < hi; i += blockDim.x) part += b.txn_ins[i];
  part = __reduce_add_sync(0xffffffffu, part);
  if ((threadIdx.x & 31) == 0) wsum[threadIdx.x >> 5] = part;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int w = 0; w < 8; ++w) t += wsum[w];
    partials[blockIdx.x] = t;
  }
  grid.sync();
  if (threadIdx.x == 0) {
    uint32_t off = 0;
    for (uint32_t q = 0; q < blockIdx.x; ++q) off += partials[q];
    carry = off;
    if (blockIdx.x == gridDim.x - 1) {
      uint32_t tot = off;
      for (uint32_t q = blockIdx.x; q < gridDim.x; ++q) tot += partials[q];
      b.txn_ins[n] = tot;
    }
  }
  __syncthreads();
  const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (uint32_t base = lo; base < hi; base += blockDim.x) {  // 256 at a time, carried across rounds
    const uint32_t i = base + threadIdx.x;
    const uint32_t v = i < hi ? b.txn_ins[i] : 0u;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= (uint32_t)o) x += y;
    }
    __syncthreads();
    if (lane == 31) wsum[wid] = x;
    __syncthreads();
    uint32_t before = carry, round = 0;
    for (uint32_t w = 0; w < 8; ++w) {
      if (w < wid) before += wsum[w];
      round += wsum[w];
    }
    if (i < hi) b.txn_ins[i] = before + x - v;
    __syncthreads();
    if (threadIdx.x == 0) carry += round;
  }
  grid.sync();
  if (blockIdx.x == 0 && threadIdx.x == 0)
    capacity_body(n_tables, b.ins_tables, b.txn_ins + n, b.base, b.reserve, b.err);
  grid.sync();
  ops_claim_body(b);
  grid.sync();
  if (run_exec) ops_exec_body<true>(b, filter);  // (fused front end: only the INSERT list is populated)
}
__global__ void __launch_bounds__(256) k_ops_insert_tail(uint32_t n_tables, BatchDev b, bool filter,
                                                         uint32_t* partials) {
  cg::grid_group grid = cg::this_grid();
  ops_insert_tail_body(n_tables, b, filter, partials, grid);
}

void launch_ops_insert_tail(uint32_t n_tables, const BatchDev& b, bool filter, uint32_t* partials, cudaStream_t s) {
  static int per_sm = 0, sms = 0;
  if (!per_sm) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_ops_insert_tail, 256, 0) != cudaSuccess || per_sm < 1)
      per_sm = 1;
  }
  const uint32_t want = std::max<uint32_t>(1, (b.n_txns + 1023) / 1024);
  const uint32_t grid = std::min<uint32_t>(std::min<uint32_t>(want, (uint32_t)(per_sm * sms)), 4096);  // partials[4096]
  uint32_t nt = n_tables;
  BatchDev bb = b;
  bool f = filter;
  void* args[] = {&nt, &bb, &f, &partials};
  cudaLaunchCooperativeKernel((const void*)k_ops_insert_tail, dim3(grid), dim3(256), args, 0, s);
  note_launch();
}

void launch_ops_exec(const BatchDev& b, bool grouped, bool filter, cudaStream_t s) {
  uint64_t warps = (b.n_ops + NKINDS * 32 + 31) / 32;
  uint64_t blocks = (warps + 7) / 8;
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (!blocks) return;
  if (grouped)
    k_ops_exec<true><<<(unsigned)blocks, 256, 0, s>>>(b, filter);
  else
    k_ops_exec<false><<<(unsigned)blocks, 256, 0, s>>>(b, filter);
  note_launch();
}

// ---- K-detect: per txn, OR of the unit tests over its ops ------------------------------
// PART: partitioned -- only this partition's ops / keys are checked and the verdict goes
// to lflag (conflict*2 | user_abort) for the exchange; otherwise it is final (status).
// the RAW/WAW(/WAR) bits of op i of txn r (PART: only this partition's keys of a SCAN)
template <bool PART>
__device__ __forceinline__ uint32_t ops_detect_op(const BatchDev& b, uint32_t i, uint32_t r, uint32_t dmask) {
  const uint64_t u = b.uref[i];
  const uint64_t chk = u >> 62;
  if (chk == CHK_NONE) return 0;
  const uint32_t t = (u >> 40) & 0xFF;
  const DevTable& T = c_tabs[t];
  uint32_t bits = 0;
  if (chk == CHK_SCAN) {  // phantom-safe: every key of the range is a read (R8)
    const ltpg_op o = load_op(b.ops, i);
    if (!T.n_groups) return 0;
    const uint32_t gs = (o.col != LTPG_COL_COUNT && col_group(T, o.col) != LTPG_STATIC) ? col_group(T, o.col) : 0;
    for (uint64_t k = o.key; k < o.key + o.aux && !(bits & CF_RAW); ++k) {
      if (PART && !owns_key(b, T, k)) continue;
      uint32_t row, claim;
      lookup(T, t, dmask, k, row, claim);
      if (row != ROW_NONE) bits |= unit_bits(T, gs, row, ACC_READ, r, b_epoch(b));
      else if (claim != ROW_NONE) bits |= unit_bits(T, 0, claim, ACC_READ, r, b_epoch(b));
    }
    return bits;
  }
  if (u & UREF_RECHECK) {  // absent at execution (fused path): an INSERT may have claimed it since
    const ltpg_op o = load_op(b.ops, i);
    uint32_t row, claim;
    lookup(T, t, dmask, o.key, row, claim);
    return claim != ROW_NONE ? unit_bits(T, 0, claim, ACC_READ, r, b_epoch(b)) : 0u;
  }
  const uint32_t row = (uint32_t)u;
  const uint32_t acc = chk == CHK_A ? ACC_ADD : (((u >> 59) & 1) ? ACC_WRITE : ACC_READ);
  if ((u >> 61) & 1) {
    for (uint32_t g = 0; g < T.n_groups; ++g) bits |= unit_bits(T, g, row, acc, r, b_epoch(b));
  } else {
    bits |= unit_bits(T, (u >> 32) & 0xFF, row, acc, r, b_epoch(b));
  }
  return bits;
}
template <bool PART>
__device__ __forceinline__ void ops_detect_txn(const BatchDev& b, uint32_t r) {
  const uint32_t dmask = *b.dense_live & ~*b.insdel;
  const bool reorder = b.flags & LTPG_FLAG_REORDER;
  const uint32_t b0 = b.op_begin[r], b1 = b.op_begin[r + 1];
  uint32_t bits = 0;
  for (uint32_t i = b0; i < b1 && !conflict_of(bits, reorder); ++i) {
    if (PART && !op_touches(b, load_op(b.ops, i))) continue;
    bits |= ops_detect_op<PART>(b, i, r, dmask);
  }
  const uint32_t flag = bits | (b.ua[r] ? CF_UA : 0u);
  if (PART) b.lflag[r] = (uint8_t)flag;
  else b.status[r] = status_of_bits(flag, reorder);
}
template <bool PART>
__global__ void __launch_bounds__(256) k_ops_detect(BatchDev b) {
  if (*b.err) return;
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r < b.n_txns) ops_detect_txn<PART>(b, r);
}

void launch_ops_detect(const BatchDev& b, cudaStream_t s) {
  if (b.nparts > 1)
    k_ops_detect<true><<<(b.n_txns + 255) / 256, 256, 0, s>>>(b);
  else
    k_ops_detect<false><<<(b.n_txns + 255) / 256, 256, 0, s>>>(b);
  note_launch();
}

// ---- K-wb: apply committed write sets; every INSERT releases its claim ----------------
// op i (of a committed txn, or an INSERT of any txn: its claim is released).  The ops of one txn
// touch distinct keys (R10), so they may be applied in any order and by different threads.
// EAGER: the result slot and argument are loaded together with the uref (one round trip instead
// of two on the latency-bound small path; the large-batch path loads them only for UPDATE / ADD)
template <bool EAGER = false>
__device__ __forceinline__ void ops_writeback_op(const BatchDev& b, uint32_t i, const ltpg_op& o, bool commit) {
  const uint64_t u = b.uref[i];
  long long rv = 0, av = 0;
  if (EAGER) rv = b.res[i], av = b.args[i];
  if ((u >> 62) == CHK_NONE || (u >> 62) == CHK_SCAN) return;
  const bool present = (u >> 60) & 1;
  const uint32_t row = (uint32_t)u;
  const DevTable& T = c_tabs[o.table];
  if (o.kind == LTPG_INSERT) {
    if (present) return;  // duplicate-key user abort: nothing claimed
    IdxSlot* sl = idx_slot(T, o.key);
    if (!sl) { atomicOr(b.err, ERR_EINTERNAL); return; }
    if (commit) {
      const long long arg = EAGER ? av : b.args[i];
      for (uint32_t c = 0; c < T.n_cols; ++c)
        *col_ptr_ops(T, c, row) = (long long)((unsigned long long)arg + c);
      T.rowkey[row] = o.key;
      T.valid[row] = 1;
      sl->row = row;
    }
    sl->claim = ROW_NONE;
    return;
  }
  if (!present) return;
  switch (o.kind) {
    case LTPG_UPDATE:
      *col_ptr_ops(T, o.col, row) = (long long)((unsigned long long)(EAGER ? rv : b.res[i]) +
                                                (unsigned long long)(EAGER ? av : b.args[i]));
      break;
    case LTPG_ADD:  // delayed update: commutative, order-free and exact
      atomicAdd(reinterpret_cast<unsigned long long*>(col_ptr_ops(T, o.col, row)),
                (unsigned long long)(EAGER ? av : b.args[i]));
      break;
    case LTPG_DELETE: {
      T.valid[row] = 0;
      IdxSlot* sl = idx_slot(T, o.key);
      if (sl) sl->row = ROW_NONE;
      break;
    }
    default:
      break;
  }
}
__device__ __forceinline__ void ops_writeback_txn(const BatchDev& b, uint32_t r) {
  const bool commit = b.status[r] == LTPG_ST_COMMIT;  // final verdict (after the exchange)
  if (!commit && b.txn_ins[r + 1] == b.txn_ins[r]) return;  // aborted, no claims to release
  const uint32_t b0 = b.op_begin[r], b1 = b.op_begin[r + 1];
  for (uint32_t i = b0; i < b1; ++i) {
    const ltpg_op o = load_op(b.ops, i);
    if (!commit && o.kind != LTPG_INSERT) continue;
    if (!op_touches(b, o)) continue;  // another partition's op: its uref is not ours
    ops_writeback_op(b, i, o, commit);
  }
}
// ADV (single-partition batches): the grid's last block also advances the append cursors past
// this batch's reservations and retires the dense key mapping of tables that saw INSERT or
// DELETE (what k_advance does after the write-back of every partition otherwise)
template <bool ADV>
__global__ void __launch_bounds__(256) k_ops_writeback(BatchDev b, uint32_t n_tables) {
  if (*b.err) return;  // (no block counts: the cursors stay put)
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r < b.n_txns) ops_writeback_txn(b, r);
  if (ADV && last_block(b.done) && threadIdx.x == 0 && !*(volatile uint32_t*)b.err) {
    for (uint32_t t = 0; t < n_tables; ++t) *c_tabs[t].n_rows += b.reserve[t];
    *b.dense_live &= ~*b.insdel;
  }
}

void launch_ops_writeback(const BatchDev& b, uint32_t n_tables, bool advance, cudaStream_t s) {
  if (advance)
    k_ops_writeback<true><<<(b.n_txns + 255) / 256, 256, 0, s>>>(b, n_tables);
  else
    k_ops_writeback<false><<<(b.n_txns + 255) / 256, 256, 0, s>>>(b, n_tables);
  note_launch();
}


// ---- small batches: the whole a1..a8 pipeline in ONE cooperative launch ------------------
// A batch of a few thousand txns runs each stage in a few microseconds, so per-kernel launch
// gaps were most of its latency, and one thread per txn left each thread a serial chain of its
// ops' dependent loads.  Here the stages are separated by grid-wide barriers and the op-level
// stages run one thread per op (from the per-kind lists), so a stage costs about one dependent
// memory round trip:
//   a1 validate + per-kind lists (K-group; + the batch's clears) -> INSERT tail (scan, capacity,
//   K-claim; only with INSERTs) -> a4/a5 execute every list (K-exec) -> a6 per-op RAW/WAW(/WAR)
//   bits, OR-ed into the txn's verdict byte -> {a6 status + a7 per op + cursor advance; a8 in
//   the grid's last block}.
// Same per-op code as the multi-kernel unfused path (the verdict is the OR of the ops' bits:
// conflict_of / status_of_bits are monotone in the bits), hence result-identical.  A thread
// keeps its op (list entry + record) in registers across the op stages when the grid covers
// every op.  The partition's small words (error, counters) are a per-slot set that the batch's
// result publish (k_publish) reads and clears, so they need no clearing barrier here.
// Single partition only (no exchange), no large-sized buckets (their fold is its own pass).
#ifdef LTPG_SMALL_TS
__device__ unsigned long long g_small_we[8];  // per phase: the latest end of a thread's work
#endif
// Warm-up by the blocks that hold no txns during K-group: read the op records (so K-group's
// staging loads find them in L2) and fetch every point op's row word, write mark (or index
// home slot) and argument into L2 for the op stages that follow.  Loads and prefetches only.
__device__ __forceinline__ void small_warm(const BatchDev& b, uint32_t t0, uint32_t nt) {
  const uint32_t live = *b.dense_live;
  for (uint32_t i = t0; i < b.n_ops; i += nt) {
    const ltpg_op o = load_op(b.ops, i);
    if (o.table >= MAXT || o.kind == LTPG_SCAN) continue;
    const DevTable& T = c_tabs[o.table];
    if (!T.defined) continue;
    if (o.kind != LTPG_SELECT) prefetch_l2(b.args + i);
    if (o.kind == LTPG_INSERT) continue;
    if (((live >> o.table) & 1u) && o.key - T.key_base < T.dense_n) {
      const uint32_t row = (uint32_t)(o.key - T.key_base);
      if (o.col < T.n_cols) prefetch_l2(col_ptr_ops(T, o.col, row));
      if (T.wmarks) {
        const uint32_t g = o.col < T.n_cols && col_group(T, o.col) != LTPG_STATIC ? col_group(T, o.col) : 0;
        prefetch_l2(wmark_ptr(T, g < T.n_groups ? g : 0, row));
      }
    } else if (T.idx) {
      prefetch_l2(T.idx + idx_hash(o.key, T.idx_shift));
    }
  }
}

// the p-th entry of the concatenated per-kind lists (kinds in order)
__device__ __forceinline__ unsigned long long list_entry(const BatchDev& b, uint32_t p, const uint32_t (&cnt)[NKINDS]) {
  uint32_t k = 0;
#pragma unroll
  for (int kk = 0; kk < NKINDS - 1; ++kk)
    if (k == (uint32_t)kk && p >= cnt[kk]) { p -= cnt[kk]; k = kk + 1; }
  return b.items[(uint64_t)k * b.max_ops + p];
}

__global__ void __launch_bounds__(256) k_ops_small(uint32_t n_tables, BatchDev b, bool filter, uint32_t* partials,
                                                   SmallOut o) {
  __shared__ __align__(16) ltpg_op stage[8][GROUP_STAGE];
  cg::grid_group grid = cg::this_grid();  // (the INSERT tail's barriers)
  uint32_t* bar = o.bar;  // zero at launch, cleared by the last block
  const uint32_t n = b.n_txns;
  const bool fin_block = blockIdx.x == gridDim.x - 1;  // a8 only; no op work
  const uint32_t gt = blockIdx.x * blockDim.x + threadIdx.x, gs = (gridDim.x - 1) * blockDim.x;
  const bool reorder = b.flags & LTPG_FLAG_REORDER;
#ifdef LTPG_SMALL_TS  // phase timestamps (diagnostic builds only): printed by thread 0
  unsigned long long ts[8];
  int nts = 0;
#define SMALL_TS() \
  if (gt == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(ts[nts++]))
#define WORK_END(k)                                                    \
  {                                                                    \
    __syncthreads();                                                   \
    unsigned long long t_;                                             \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));             \
    if (threadIdx.x == 0) atomicMax(g_small_we + (k), t_);             \
  }
#else
#define SMALL_TS()
#define WORK_END(k)
#endif
  SMALL_TS();
  WORK_END(7);  // the last block's start
  // a1 + per-kind lists, one thread per txn (blocks [0, ceil(n/256)) cover the batch), and the
  // batch's clears for the later stages: reservations, batch scalars (read with ld.global.nc by
  // b_epoch after the barrier below -- no SM cached their line in this launch before), user-abort
  // flags, verdict bytes
  if (blockIdx.x == 0) {
    if (threadIdx.x < MAXT) o.reserve[threadIdx.x] = 0;
    if (threadIdx.x == 0) {
      o.vars->epoch = o.host ? o.host->epoch : o.epoch;
      o.vars->clock = o.host ? o.host->clock : o.clock;
    }
  }
  if (gt < n) b.ua[gt] = 0;
  if (gt < (n + 3) / 4) reinterpret_cast<uint32_t*>(b.lflag)[gt] = 0;
  const uint32_t txn_blocks = (n + blockDim.x - 1) / blockDim.x;
#ifndef LTPG_SMALL_NO_WARM
  if (blockIdx.x >= txn_blocks)
    small_warm(b, (blockIdx.x - txn_blocks) * blockDim.x + threadIdx.x, (gridDim.x - txn_blocks) * blockDim.x);
#endif
  ops_validate_group_body<true>(n_tables, b, stage);
  WORK_END(0);
  grid_barrier(bar, 1);
  SMALL_TS();
  ops_insert_tail_body(n_tables, b, filter, partials, grid, false);  // INSERTs: scan, capacity, claims
  SMALL_TS();
  uint32_t cnt[NKINDS], total = 0;
#pragma unroll
  for (int k = 0; k < NKINDS; ++k) total += (cnt[k] = *(volatile uint32_t*)(b.kcount + k));
  const bool ok = *(volatile uint32_t*)b.err == 0;  // uniform: raised before the last barrier
  const uint32_t dmask = *b.dense_live & ~*b.insdel;
  const bool one = total <= gs;  // every op has its own thread: keep it in registers
  unsigned long long it1 = 0;
  ltpg_op op1{};
  if (ok && !fin_block) {  // a4/a5: one thread per op
    if (one) {
      if (gt < total) {
        it1 = list_entry(b, gt, cnt);
        op1 = load_op(b.ops, (uint32_t)it1);
        exec_one(b, (uint32_t)it1, (uint32_t)(it1 >> 32), op1, filter, dmask);
      }
    } else {
      for (uint32_t p = gt; p < total; p += gs) {
        const unsigned long long it = list_entry(b, p, cnt);
        exec_one(b, (uint32_t)it, (uint32_t)(it >> 32), load_op(b.ops, (uint32_t)it), filter, dmask);
      }
    }
  }
  WORK_END(2);
  grid_barrier(bar, 2);
  SMALL_TS();
  if (ok && !fin_block)  // a6: one thread per op, OR into the txn's byte
    for (uint32_t p = gt; p < total; p += gs) {
      const unsigned long long it = one ? it1 : list_entry(b, p, cnt);
      const uint32_t r = (uint32_t)(it >> 32);
      const uint32_t bits = ops_detect_op<false>(b, (uint32_t)it, r, dmask);
      if (bits) atomicOr(reinterpret_cast<uint32_t*>(b.lflag) + (r >> 2), bits << (8 * (r & 3)));
    }
  WORK_END(3);
  grid_barrier(bar, 3);
  SMALL_TS();
  auto st_of = [&](uint32_t r) { return status_of_bits(b.lflag[r] | (b.ua[r] ? CF_UA : 0u), reorder); };
  if (fin_block) {
    if (ok) finalize_block(n, o, st_of);  // a8
  } else if (ok) {
    for (uint32_t p = gt; p < total; p += gs) {  // a7: one thread per op
      const unsigned long long it = one ? it1 : list_entry(b, p, cnt);
      const uint32_t oi = (uint32_t)it;
      const ltpg_op op = one ? op1 : load_op(b.ops, oi);
      const bool commit = st_of((uint32_t)(it >> 32)) == LTPG_ST_COMMIT;
      if (commit || op.kind == LTPG_INSERT) ops_writeback_op<true>(b, oi, op, commit);
    }
    for (uint32_t r = gt; r < n; r += gs) b.status[r] = st_of(r);
    // cursors past this batch's reservations (nothing of a7 reads them; an error raised by a7
    // is internal and poisons the db)
    if (gt == 0) {
      for (uint32_t t = 0; t < n_tables; ++t)
        if (o.reserve[t]) *c_tabs[t].n_rows += o.reserve[t];
      if (*b.insdel) *b.dense_live &= ~*b.insdel;
    }
  }
  WORK_END(fin_block ? 5 : 4);
  if (!ok && fin_block && threadIdx.x < 17 && (threadIdx.x || o.write0))
    o.dsmall[threadIdx.x] = 0;  // failed batch (the error is in the partition's word): no counts
  // the last block to finish publishes the result words into the slot's mapped host words (what
  // k_publish does after the multi-kernel path) and clears the partition words for the slot's
  // next batch (which is stream-ordered after this kernel)
  __shared__ bool last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd(b.done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (last) {
    __threadfence();
    if (threadIdx.x < 17)
      o.host_small[threadIdx.x] = reinterpret_cast<volatile uint32_t*>(o.dsmall)[threadIdx.x] |
                                  (threadIdx.x == 0 ? *reinterpret_cast<volatile uint32_t*>(b.err) : 0u);
    __syncthreads();
    if (threadIdx.x < 16) b.err[threadIdx.x] = 0;  // err .. done
    if (threadIdx.x == 0) *o.bar = 0;
  }
#ifdef LTPG_SMALL_TS
  SMALL_TS();
  if (gt == 0) {
    volatile unsigned long long* we = g_small_we;
    printf("k_ops_small n=%u ops=%u grid=%u ns: group %llu ins %llu exec %llu detect %llu fin+wb %llu | "
           "last block start +%lld | work: group %lld exec %lld detect %lld wb %lld fin %lld\n", n, total,
           gridDim.x, ts[1] - ts[0], ts[2] - ts[1], ts[3] - ts[2], ts[4] - ts[3], ts[5] - ts[4],
           (long long)(we[7] - ts[0]), (long long)(we[0] - ts[0]), (long long)(we[2] - ts[2]),
           (long long)(we[3] - ts[3]), (long long)(we[4] - ts[4]), (long long)(we[5] - ts[4]));
    for (int k = 0; k < 8; ++k) we[k] = 0;
  }
#endif
#undef SMALL_TS
#undef WORK_END
}

uint32_t ops_small_max_txns() { return 16384; }

void launch_ops_small(uint32_t n_tables, const BatchDev& b, bool filter, uint32_t* partials,
                      unsigned long long* reserve, BatchVars* vars, const volatile BatchVars* host, uint32_t epoch,
                      long long clock, uint32_t* commit_bits, uint32_t* dsmall, bool write0, uint32_t* abort_out,
                      uint32_t* n_out2, volatile uint32_t* host_small, uint32_t* bar, cudaStream_t s) {
  static int per_sm = 0, sms = 0;
  if (!per_sm) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_ops_small, 256, 0) != cudaSuccess || per_sm < 1)
      per_sm = 1;
  }
  uint32_t nt = n_tables;
  BatchDev bb = b;
  bool f = filter;
  SmallOut so{reserve, vars, host, epoch, clock, commit_bits, dsmall, abort_out, n_out2, host_small, write0, bar};
  void* args[] = {&nt, &bb, &f, &partials, &so};
  // one thread per txn for K-group, one per op for the op stages (grid-stride beyond), + the a8
  // block; co-resident
  const uint32_t want = std::max<uint32_t>((b.n_txns + 255) / 256, (b.n_ops + 255) / 256) + 1;
  const uint32_t grid = std::max<uint32_t>(2, std::min<uint32_t>(want, (uint32_t)(per_sm * sms)));
  cudaLaunchCooperativeKernel((const void*)k_ops_small, dim3(grid), dim3(256), args, 0, s);
  note_launch();
}

}  // namespace ltpg
