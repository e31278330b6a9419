// Shared kernels: deterministic exclusive scan, result finalisation (commit
// bitmask via __ballot_sync, abort-list compaction), index build, capacity and
// append-cursor bookkeeping.
#include <algorithm>

#include "ltpg_internal.cuh"

namespace ltpg {

uint64_t g_kernel_launches = 0;
LTPG_DEFINE_TABLE_UPLOAD(upload_tables_common)

constexpr int SCAN_THREADS = 256;
constexpr int SCAN_ITEMS = 16;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;  // 4096 elements per block

// Block-wide exclusive scan of one value per thread; returns the block total.
template <class T>
__device__ __forceinline__ T block_excl_scan(T v, T& total) {
  __shared__ T warp_tot[SCAN_THREADS / 32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  T x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) warp_tot[wid] = x;
  __syncthreads();
  if (wid == 0) {
    T t = lane < SCAN_THREADS / 32 ? warp_tot[lane] : T(0);
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      T y = __shfl_up_sync(0xffffffffu, t, o);
      if (lane >= o) t += y;
    }
    if (lane < SCAN_THREADS / 32) warp_tot[lane] = t;  // inclusive
  }
  __syncthreads();
  total = warp_tot[SCAN_THREADS / 32 - 1];
  T base = wid ? warp_tot[wid - 1] : T(0);
  __syncthreads();
  return base + x - v;
}

template <class T>
__global__ void k_scan_reduce(const T* __restrict__ in, uint32_t n, T* __restrict__ sums, const uint32_t* skip) {
  if (skip && !*skip) return;
  const uint64_t base = (uint64_t)blockIdx.x * SCAN_TILE;
  T s = 0;
#pragma unroll
  for (int k = 0; k < SCAN_ITEMS; ++k) {
    uint64_t i = base + (uint64_t)k * SCAN_THREADS + threadIdx.x;
    if (i < n) s += in[i];
  }
  T tot;
  block_excl_scan<T>(s, tot);
  if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

// single block: exclusive scan of the block sums (nb <= SCAN_TILE); sums[nb] = total
template <class T>
__global__ void k_scan_top(T* sums, uint32_t nb, const uint32_t* skip) {
  if (skip && !*skip) return;
  T v[SCAN_ITEMS];
  T s = 0;
#pragma unroll
  for (int k = 0; k < SCAN_ITEMS; ++k) {
    uint32_t i = threadIdx.x * SCAN_ITEMS + k;
    v[k] = i < nb ? sums[i] : T(0);
    s += v[k];
  }
  T tot;
  T off = block_excl_scan<T>(s, tot);
#pragma unroll
  for (int k = 0; k < SCAN_ITEMS; ++k) {
    uint32_t i = threadIdx.x * SCAN_ITEMS + k;
    if (i < nb) sums[i] = off;
    off += v[k];
  }
  if (threadIdx.x == 0) sums[nb] = tot;
}

template <class T>
__global__ void k_scan_down(const T* __restrict__ in, T* __restrict__ out, uint32_t n,
                            const T* __restrict__ sums, uint32_t nb, const uint32_t* skip) {
  if (skip && !*skip) {  // every input is zero (in-place scan): only the total is missing
    if (blockIdx.x == 0 && threadIdx.x == 0) out[n] = 0;
    return;
  }
  // each thread owns SCAN_ITEMS consecutive elements of the tile (stable order)
  const uint64_t base = (uint64_t)blockIdx.x * SCAN_TILE + (uint64_t)threadIdx.x * SCAN_ITEMS;
  T v[SCAN_ITEMS];
  T s = 0;
#pragma unroll
  for (int k = 0; k < SCAN_ITEMS; ++k) {
    uint64_t i = base + k;
    v[k] = i < n ? in[i] : T(0);
    s += v[k];
  }
  T tot;
  T off = block_excl_scan<T>(s, tot) + sums[blockIdx.x];
#pragma unroll
  for (int k = 0; k < SCAN_ITEMS; ++k) {
    uint64_t i = base + k;
    if (i < n) out[i] = off;
    off += v[k];
  }
  if (blockIdx.x == nb - 1 && threadIdx.x == 0) out[n] = sums[nb];
}

size_t scan_scratch_words(uint32_t n) { return 2 * ((n + SCAN_TILE - 1) / SCAN_TILE + 2); }

// out[0..n) = exclusive prefix sums of in, out[n] = total.  Deterministic.  scratch holds
// scan_scratch_words(n) u32 words (enough for 64-bit sums).
template <class T>
static void scan_exclusive(const T* in, T* out, uint32_t n, void* scratch_v, cudaStream_t s,
                           const uint32_t* skip = nullptr) {
  T* scratch = static_cast<T*>(scratch_v);
  if (n == 0) {
    cudaMemsetAsync(out, 0, sizeof(T), s);
    return;
  }
  uint32_t nb = (n + SCAN_TILE - 1) / SCAN_TILE;  // <= SCAN_TILE blocks (n <= 16.7M)
  k_scan_reduce<T><<<nb, SCAN_THREADS, 0, s>>>(in, n, scratch, skip);
  k_scan_top<T><<<1, SCAN_THREADS, 0, s>>>(scratch, nb, skip);
  k_scan_down<T><<<nb, SCAN_THREADS, 0, s>>>(in, out, n, scratch, nb, skip);
  note_launch(3);
}

void scan_exclusive_u32(const uint32_t* in, uint32_t* out, uint32_t n, uint32_t* scratch, cudaStream_t s,
                        const uint32_t* skip_if_zero) {
  scan_exclusive<uint32_t>(in, out, n, scratch, s, skip_if_zero);
}
void scan_exclusive_u64(const unsigned long long* in, unsigned long long* out, uint32_t n, uint32_t* scratch,
                        cudaStream_t s) {
  scan_exclusive<unsigned long long>(in, out, n, scratch, s);
}

// Result finalisation: commit bitmask (one __ballot_sync word per warp), conflict
// flags for the abort list, per-status counts.
__global__ void k_finalize(const uint8_t* __restrict__ status, uint32_t n, uint32_t* __restrict__ commit_bits,
                           uint32_t* __restrict__ flags, uint32_t* __restrict__ counts,
                           const uint32_t* __restrict__ err) {
  __shared__ uint32_t red[3];
  if (*err) return;
  if (threadIdx.x < 3) red[threadIdx.x] = 0;
  __syncthreads();
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  const uint8_t st = r < n ? status[r] : 0xFF;
  const uint32_t bits = __ballot_sync(0xffffffffu, st == LTPG_ST_COMMIT);
  if ((threadIdx.x & 31) == 0 && r < n) commit_bits[r >> 5] = bits;
  if (r < n) flags[r] = st == LTPG_ST_CONFLICT;
  const uint32_t na = __popc(__ballot_sync(0xffffffffu, st == LTPG_ST_CONFLICT));
  const uint32_t nu = __popc(__ballot_sync(0xffffffffu, st == LTPG_ST_USER_ABORT));
  if ((threadIdx.x & 31) == 0) {  // block-level totals: one global atomic per block and counter
    atomicAdd(red + 0, __popc(bits));
    atomicAdd(red + 1, na);
    atomicAdd(red + 2, nu);
  }
  __syncthreads();
  if (threadIdx.x < 3 && red[threadIdx.x]) atomicAdd(counts + threadIdx.x, red[threadIdx.x]);
}

void launch_finalize(const uint8_t* status, uint32_t n, uint32_t* commit_bits, uint32_t* flags, uint32_t* counts,
                     const uint32_t* err, cudaStream_t s) {
  if (!n) return;
  k_finalize<<<(n + 1023) / 1024, 1024, 0, s>>>(status, n, commit_bits, flags, counts, err);
  note_launch();
}

// a8 in one pass: commit bitmask, per-status counts and the abort list (ascending ranks) with
// a decoupled look-back scan over 1024-txn tiles.  Tile ids come from a counter (reset per
// batch), so every tile a block waits for belongs to a block that is already running.  Tile
// state word: [63:32] batch epoch | [31:30] 1 = aggregate, 2 = inclusive prefix | [29:0] value.
constexpr uint32_t FC_TILE = 1024;
__global__ void __launch_bounds__(256) k_finalize_compact(const uint8_t* __restrict__ status, uint32_t n,
                                                          uint32_t* __restrict__ commit_bits, uint32_t* counts,
                                                          const uint32_t* err, uint32_t* __restrict__ out,
                                                          uint32_t* n_out, uint32_t* n_out2,
                                                          unsigned long long* tile_state, uint32_t* tile_ctr,
                                                          const BatchVars* __restrict__ vars) {
  __shared__ uint32_t tile_s, wsum[8], red[3], base_s;
  (void)err;  // no early exit: write-back may raise the error word concurrently, and a block
              // that skipped its tile would leave its successors waiting forever
  if (threadIdx.x == 0) tile_s = atomicAdd(tile_ctr, 1u);
  if (threadIdx.x < 3) red[threadIdx.x] = 0;
  __syncthreads();
  const uint32_t tile = tile_s, lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t r0 = tile * FC_TILE + 4 * threadIdx.x;
  uint8_t st[4];
  if (r0 + 3 < n) {
    const uchar4 v = *reinterpret_cast<const uchar4*>(status + r0);
    st[0] = v.x, st[1] = v.y, st[2] = v.z, st[3] = v.w;
  } else {
#pragma unroll
    for (uint32_t j = 0; j < 4; ++j) st[j] = r0 + j < n ? status[r0 + j] : 0xFF;
  }
  uint32_t nib = 0, nc = 0, nu = 0;
#pragma unroll
  for (uint32_t j = 0; j < 4; ++j) {
    nib |= (st[j] == LTPG_ST_COMMIT ? 1u : 0u) << j;
    nc += st[j] == LTPG_ST_CONFLICT;
    nu += st[j] == LTPG_ST_USER_ABORT;
  }
  // commit bits: 8 lanes (32 txns) per word
  uint32_t word = nib << (4 * (lane & 7));
  word |= __shfl_xor_sync(0xffffffffu, word, 1);
  word |= __shfl_xor_sync(0xffffffffu, word, 2);
  word |= __shfl_xor_sync(0xffffffffu, word, 4);
  if ((lane & 7) == 0 && r0 < n) commit_bits[r0 >> 5] = word;
  // block-wide exclusive scan of the per-thread conflict counts (rank order)
  uint32_t x = nc;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  const uint32_t ncw = __reduce_add_sync(0xffffffffu, nc), nuw = __reduce_add_sync(0xffffffffu, nu);
  const uint32_t nbw = __reduce_add_sync(0xffffffffu, __popc(nib));
  if (lane == 31) wsum[wib] = x;
  if (lane == 0) {
    atomicAdd(red + 0, nbw);
    atomicAdd(red + 1, ncw);
    atomicAdd(red + 2, nuw);
  }
  __syncthreads();
  uint32_t before = 0, agg = 0;
#pragma unroll
  for (uint32_t w = 0; w < 8; ++w) {
    if (w < wib) before += wsum[w];
    agg += wsum[w];
  }
  if (threadIdx.x < 3 && red[threadIdx.x]) atomicAdd(counts + threadIdx.x, red[threadIdx.x]);
  if (threadIdx.x == 0) {  // decoupled look-back
    const uint32_t epoch = vars->epoch;
    const unsigned long long tag = (unsigned long long)epoch << 32;
    volatile unsigned long long* vs = tile_state;
    uint32_t base = 0;
    if (tile == 0) {
      vs[0] = tag | (2ull << 30) | agg;
    } else {
      vs[tile] = tag | (1ull << 30) | agg;
      for (int64_t j = (int64_t)tile - 1; j >= 0;) {
        const unsigned long long v = vs[j];
        const uint32_t fl = (v >> 32) == epoch ? (uint32_t)(v >> 30) & 3u : 0u;
        if (!fl) continue;  // predecessor not published yet
        base += (uint32_t)v & 0x3FFFFFFFu;
        if (fl == 2) break;
        --j;
      }
      vs[tile] = tag | (2ull << 30) | (base + agg);
    }
    base_s = base;
    if ((tile + 1) * FC_TILE >= n) {  // the last tile knows the total
      *n_out = base + agg;
      if (n_out2) *n_out2 = base + agg;
    }
  }
  __syncthreads();
  uint32_t o = base_s + before + x - nc;
#pragma unroll
  for (uint32_t j = 0; j < 4; ++j)
    if (st[j] == LTPG_ST_CONFLICT) out[o++] = r0 + j;
}

void launch_finalize_compact(const uint8_t* status, uint32_t n, uint32_t* commit_bits, uint32_t* counts,
                             const uint32_t* err, uint32_t* out, uint32_t* n_out, uint32_t* n_out2,
                             unsigned long long* tile_state, uint32_t* tile_ctr, const BatchVars* vars, cudaStream_t s) {
  if (!n) return;
  cudaMemsetAsync(tile_ctr, 0, sizeof(uint32_t), s);
  k_finalize_compact<<<(n + FC_TILE - 1) / FC_TILE, 256, 0, s>>>(status, n, commit_bits, counts, err, out, n_out,
                                                                 n_out2, tile_state, tile_ctr, vars);
  note_launch();
}

// packed TPC-C parameter blocks -> fixed 128-byte blocks (zero-filled tails); one warp per
// 8 txns, 16-byte lanes
__global__ void k_unpack_params(const uint8_t* __restrict__ packed, const uint32_t* __restrict__ offs, uint32_t n,
                                uint8_t* __restrict__ params, uint32_t* err) {
  const uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  const uint32_t r = (uint32_t)(g >> 3), q = (uint32_t)(g & 7);  // txn, 16-byte quarter
  if (r >= n) return;
  const uint32_t o0 = offs[r], o1 = offs[r + 1];
  if (o1 < o0 || o1 - o0 > LTPG_PARAM_BYTES) {
    if (q == 0) atomicOr(err, ERR_EINVAL);
    return;
  }
  uint8_t v[16];
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    const uint32_t at = q * 16 + k;
    v[k] = at < o1 - o0 ? packed[o0 + at] : 0;
  }
  *reinterpret_cast<uint4*>(params + 128ull * r + 16 * q) = *reinterpret_cast<const uint4*>(v);
}

void launch_unpack_params(const uint8_t* packed, const uint32_t* offs, uint32_t n, uint8_t* params, uint32_t* err,
                          cudaStream_t s) {
  if (!n) return;
  k_unpack_params<<<(unsigned)((8ull * n + 255) / 256), 256, 0, s>>>(packed, offs, n, params, err);
  note_launch();
}

// LTPG_BATCH_COMPACT_PARAMS (include/ltpg.h): compact TPC-C records -> fixed 128-byte blocks.
// One warp per 32 txns: the warp's records (contiguous bytes) are staged in shared memory, each
// lane decodes its own record into a block in shared memory, and the warp stores its 4 KB of
// blocks with coalesced 16-byte stores.
constexpr int UC_WARPS = 4;
__device__ __forceinline__ uint32_t ld_u16(const uint8_t* p) { return (uint32_t)p[0] | (uint32_t)p[1] << 8; }
__global__ void __launch_bounds__(32 * UC_WARPS) k_unpack_compact(const uint8_t* __restrict__ packed,
                                                                  const uint32_t* __restrict__ offs,
                                                                  const uint8_t* __restrict__ types, uint32_t n,
                                                                  uint8_t* __restrict__ params, uint32_t* err) {
  __shared__ __align__(16) uint8_t in[UC_WARPS][32 * 128 + 32];
  // decoded blocks, rows padded to 144 bytes: with a 128-byte stride every lane's row started
  // in the same bank (32-way conflicts on each decode store)
  constexpr uint32_t OROW = 144;
  __shared__ __align__(16) uint8_t out[UC_WARPS][32 * OROW];
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t r0 = (blockIdx.x * UC_WARPS + wib) * 32;
  if (r0 >= n) return;
  const uint32_t cnt = min(32u, n - r0);
  const uint32_t lo = offs[r0], hi = offs[r0 + cnt], end = offs[n];
  if (hi < lo || hi - lo > 32 * 128 || hi > end) {
    if (lane == 0) atomicOr(err, ERR_EINVAL);
    return;
  }
  // stage [a0, hi) with 16-byte loads where aligned and inside the buffer, bytes otherwise
  const uint32_t a0 = lo & ~15u, nch = (hi - a0 + 15) / 16;
  const bool vec = ((uintptr_t)packed & 15) == 0;
  for (uint32_t c = lane; c < nch; c += 32) {
    const uint32_t at = a0 + 16 * c;
    if (vec && at + 16 <= end) {
      *reinterpret_cast<uint4*>(in[wib] + 16 * c) = *reinterpret_cast<const uint4*>(packed + at);
    } else {
      for (uint32_t k = 0; k < 16; ++k) in[wib][16 * c + k] = at + k < end ? packed[at + k] : 0;
    }
  }
  uint4* ob = reinterpret_cast<uint4*>(out[wib] + OROW * lane);
#pragma unroll
  for (int k = 0; k < 8; ++k) ob[k] = make_uint4(0, 0, 0, 0);
  __syncwarp();
  bool bad = false;
  if (lane < cnt) {
    const uint32_t r = r0 + lane, b0 = offs[r], b1 = offs[r + 1];
    const uint8_t* q = in[wib] + (b0 - a0);
    uint8_t* o = out[wib] + OROW * lane;
    const uint32_t len = b1 - b0;
    if (b1 < b0 || b0 < lo || b1 > hi || len > 128) {
      bad = true;
    } else if (types[r] == 0) {  // NewOrder: 8-byte header, 22-bit lines, u16 supply warehouses
      const uint32_t nl = len >= 8 ? q[3] : 0, nrem = len >= 8 ? q[7] : 0;
      const uint32_t lb = (22 * nl + 7) / 8;  // bytes of the line bit stream
      if (len < 8 || nl > 15 || len != 8 + lb + 2 * nrem) {
        bad = true;
      } else {
        {  // header bytes 0-6 (byte 7 stays 0) as one 8-byte store
          unsigned long long h = 0;
#pragma unroll
          for (int k = 0; k < 7; ++k) h |= (unsigned long long)q[k] << (8 * k);
          *reinterpret_cast<unsigned long long*>(o) = h;
        }
        const uint32_t w = ld_u16(q);
        uint32_t k = 0;
        for (uint32_t l = 0; l < nl; ++l) {
          // line l: bits 22 l .. 22 l + 21, inside the 4 bytes from byte 22 l / 8 (bytes past the
          // record are staged too -- the stage keeps 32 bytes of slack -- and masked off here)
          const uint8_t* L = q + 8 + (22 * l >> 3);
          const uint32_t v = ((ld_u16(L) | ld_u16(L + 2) << 16) >> ((22 * l) & 7)) & 0x3FFFFFu;
          uint32_t sw = w;
          if ((v >> 21) & 1u) {
            if (k < nrem) sw = ld_u16(q + 8 + lb + 2 * k);
            ++k;
          }
          // u32 i | u16 supply_w | u8 qty | 0, one 8-byte store
          *reinterpret_cast<uint2*>(o + 8 + 8 * l) = make_uint2(v & 0x1FFFFu, (sw & 0xFFFFu) | (((v >> 17) & 15u) + 1) << 16);
        }
        if (k != nrem) bad = true;
      }
    } else if (types[r] == 1) {  // Payment: 12 header bytes + u32 amount
      if (len != 16) {
        bad = true;
      } else {
        for (int k = 0; k < 12; ++k) o[k] = q[k];
        for (int k = 0; k < 4; ++k) o[16 + k] = q[12 + k];  // zero-extended to the i64 at 16
      }
    } else {
      for (uint32_t k = 0; k < len; ++k) o[k] = q[k];
    }
  }
  if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(err, ERR_EINVAL);
  __syncwarp();
  for (uint32_t c = lane; c < cnt * 8; c += 32)
    *reinterpret_cast<uint4*>(params + 128ull * r0 + 16 * c) =
        *reinterpret_cast<const uint4*>(out[wib] + OROW * (c >> 3) + 16 * (c & 7));
}

void launch_unpack_compact(const uint8_t* packed, const uint32_t* offs, const uint8_t* types, uint32_t n,
                           uint8_t* params, uint32_t* err, cudaStream_t s) {
  if (!n) return;
  const uint32_t warps = (n + 31) / 32;
  k_unpack_compact<<<(warps + UC_WARPS - 1) / UC_WARPS, 32 * UC_WARPS, 0, s>>>(packed, offs, types, n, params, err);
  note_launch();
}

// LTPG_RESULT_COMMITTED_READS: the 4 result slots of every committed txn, packed in rank order,
// written straight into the caller's (host-mapped or device) buffer.  One block computes the
// exclusive prefix of the commit-bitmask words' popcounts (each warp a contiguous segment read
// with coalesced loads, 8 in flight per lane; the per-thread sequential walk of 32 words it
// replaces was 54 us at 2^20 txns), then each block of the gather compacts its committed txns'
// slots in shared memory and stores them as one contiguous run of 16-byte stores (one thread per
// committed txn storing into host-mapped memory made scattered small PCIe writes: 108 us).
__global__ void __launch_bounds__(1024) k_commit_prefix(const uint32_t* __restrict__ bits, uint32_t nw,
                                                        uint32_t* __restrict__ pre) {
  __shared__ uint32_t wsum[32];
  const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const uint32_t seg = (nw + 1023) / 1024 * 32;  // words per warp, a multiple of 32
  const uint32_t w0 = wid * seg;
  uint32_t t = 0;
#pragma unroll 8
  for (uint32_t k = lane; k < seg; k += 32) t += w0 + k < nw ? __popc(bits[w0 + k]) : 0u;
  t = __reduce_add_sync(0xffffffffu, t);
  if (lane == 0) wsum[wid] = t;
  __syncthreads();
  if (wid == 0) {
    const uint32_t v = wsum[lane];
    uint32_t s = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= (uint32_t)o) s += y;
    }
    wsum[lane] = s - v;
  }
  __syncthreads();
  uint32_t carry = wsum[wid];
  for (uint32_t k = 0; k < seg; k += 32) {
    const uint32_t w = w0 + k + lane;
    const uint32_t v = w < nw ? __popc(bits[w]) : 0u;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= (uint32_t)o) x += y;
    }
    if (w < nw) pre[w] = carry + x - v;
    carry += __shfl_sync(0xffffffffu, x, 31);
  }
}
constexpr uint32_t CG_TXNS = 1024;  // txns per gather block (32 bitmask words)
__global__ void __launch_bounds__(CG_TXNS) k_commit_gather(const uint32_t* __restrict__ bits,
                                                          const uint32_t* __restrict__ pre, uint32_t n,
                                                          const long long* __restrict__ res, long long* out) {
  __shared__ __align__(16) long long buf[CG_TXNS * 4];
  __shared__ uint32_t base0, cnt;
  const uint32_t r = blockIdx.x * CG_TXNS + threadIdx.x;
  const uint32_t w = r < n ? bits[r >> 5] : 0u, b = r & 31;
  if (threadIdx.x == 0) {
    const uint32_t wf = blockIdx.x * (CG_TXNS / 32), wl = min(wf + CG_TXNS / 32, (n + 31) / 32) - 1;
    base0 = pre[wf];
    cnt = pre[wl] + __popc(bits[wl]) - pre[wf];
  }
  __syncthreads();
  if ((w >> b) & 1u) {  // committed: its slots at its rank among the block's committed txns
    const uint32_t i = pre[r >> 5] + __popc(w & ((1u << b) - 1u)) - base0;
    const longlong2 a = *reinterpret_cast<const longlong2*>(res + 4ull * r);
    const longlong2 c = *reinterpret_cast<const longlong2*>(res + 4ull * r + 2);
    reinterpret_cast<longlong2*>(buf + 4 * i)[0] = a;
    reinterpret_cast<longlong2*>(buf + 4 * i)[1] = c;
  }
  __syncthreads();
  longlong2* o = reinterpret_cast<longlong2*>(out + 4ull * base0);
  for (uint32_t j = threadIdx.x; j < 2 * cnt; j += blockDim.x) o[j] = reinterpret_cast<const longlong2*>(buf)[j];
}

void launch_committed_reads(const uint32_t* bits, uint32_t n, const long long* res, long long* out, uint32_t* pre,
                            cudaStream_t s) {
  if (!n) return;
  const uint32_t nw = (n + 31) / 32;
  k_commit_prefix<<<1, 1024, 0, s>>>(bits, nw, pre);
  k_commit_gather<<<(n + CG_TXNS - 1) / CG_TXNS, CG_TXNS, 0, s>>>(bits, pre, n, res, out);
  note_launch(2);
}

// LTPG_BATCH_TID_RANGE: tid[i] = t0 + i
__global__ void k_fill_tid(unsigned long long* tid, uint32_t n, unsigned long long t0) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) tid[i] = t0 + i;
}
void launch_fill_tid(unsigned long long* tid, uint32_t n, unsigned long long t0, cudaStream_t s) {
  if (!n) return;
  k_fill_tid<<<std::min<uint32_t>((n + 255) / 256, 148 * 8), 256, 0, s>>>(tid, n, t0);
  note_launch();
}

// LTPG_BATCH_CARRY_ABORTS: the previous batch's conflict aborts (abort[0..nc), ascending ranks) ->
// the first nc txns of this batch, with their original TIDs, types and 128-byte blocks.  One
// warp per carried txn: lanes move the block as 32 coalesced 4-byte words.
__global__ void __launch_bounds__(256) k_carry(const unsigned long long* __restrict__ ptid,
                                               const uint8_t* __restrict__ ptype, const uint8_t* __restrict__ pparams,
                                               const uint32_t* __restrict__ abort, uint32_t nc,
                                               unsigned long long* __restrict__ tid, uint8_t* __restrict__ type,
                                               uint8_t* __restrict__ params) {
  // 32 carried txns per warp and step: one coalesced load of their abort-list entries, then their
  // 128-byte blocks moved 4 at a time (8 lanes x 16 bytes each), every load of the step in flight
  // together (one txn per warp and step made each a list -> block round-trip chain: 105 us at
  // ~950 K carried txns)
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t nwarps = gridDim.x * (blockDim.x >> 5);
  for (uint32_t w0 = (blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32; w0 < nc; w0 += nwarps * 32) {
    const uint32_t j = w0 + lane;
    const uint32_t r = j < nc ? abort[j] : 0u;
    if (j < nc) {
      tid[j] = ptid[r];
      type[j] = ptype[r];
    }
#pragma unroll
    for (uint32_t k = 0; k < 8; ++k) {
      const uint32_t t = 4 * k + (lane >> 3);
      const uint32_t rr = __shfl_sync(0xffffffffu, r, t);
      if (w0 + t < nc)
        reinterpret_cast<uint4*>(params + 128ull * (w0 + t))[lane & 7] =
            reinterpret_cast<const uint4*>(pparams + 128ull * rr)[lane & 7];
    }
  }
}

void launch_carry(const unsigned long long* ptid, const uint8_t* ptype, const uint8_t* pparams, const uint32_t* abort,
                  uint32_t nc, unsigned long long* tid, uint8_t* type, uint8_t* params, cudaStream_t s) {
  if (!nc) return;
  k_carry<<<std::min<uint32_t>((nc + 255) / 256, 148 * 8), 256, 0, s>>>(ptid, ptype, pparams, abort, nc, tid, type, params);
  note_launch();
}

// abort list: ranks of conflict-aborted txns in ascending order (stable compaction)
// abort list (ascending ranks) and its length (n_out[0], and n_out2[0] when not null)
__global__ void k_compact(const uint32_t* __restrict__ flags, const uint32_t* __restrict__ offs, uint32_t n,
                          uint32_t* __restrict__ out, uint32_t* n_out, uint32_t* n_out2) {
  uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r < n && flags[r]) out[offs[r]] = r;
  if (r == 0) {
    const uint32_t tot = n ? offs[n] : 0u;
    *n_out = tot;
    if (n_out2) *n_out2 = tot;
  }
}

void launch_compact(const uint32_t* flags, const uint32_t* offs, uint32_t n, uint32_t* out, uint32_t* n_out,
                    uint32_t* n_out2, cudaStream_t s) {
  k_compact<<<n ? (n + 255) / 256 : 1, 256, 0, s>>>(flags, offs, n, out, n_out, n_out2);
  note_launch();
}

// ---- NEXT-3: large-sized bucket -> unit mark (min over the bucket's su sub-slots) ----------
// One warp per (unit, chunk of 1024 sub-slots) -- each lane reads 32 sub-slots, coalesced --
// and the chunk minima meet in the unit's word with atomicMin.  Older epochs carry larger tag
// bytes, so a stale word or sub-slot never hides a mark of this batch, and mark_rank ignores
// it when nothing of this batch is there.  Bucket (gi, row) belongs to word gi*capacity + row.
__global__ void __launch_bounds__(256) k_bucket_reduce(const mark_t* __restrict__ sub, mark_t* word, uint32_t groups,
                                                       uint32_t rows, uint64_t capacity, uint32_t stride,
                                                       const uint16_t* d_su, uint32_t t) {
  const uint32_t su = d_su[t];  // this batch's bucket size (<= stride, the allocated one)
  if (su <= 1) return;          // standard-sized this batch: the marks are in the words already
  const uint32_t per = (su + 1023) / 1024;
  const uint64_t units = (uint64_t)groups * rows;
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t c = blockIdx.x * (uint64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); c < units * per; c += nwarps) {
    const uint64_t u = c / per;
    const uint32_t j0 = (uint32_t)(c % per) * 1024u;
    const uint32_t j1 = min(su, j0 + 1024u);
    mark_t m = 0xFFFFFFFFu;
    for (uint32_t j = j0 + lane; j < j1; j += 32) m = min(m, __ldcg(sub + u * stride + j));
    m = __reduce_min_sync(0xffffffffu, m);
    if (lane == 0 && m != 0xFFFFFFFFu) atomicMin(word + (u / rows) * capacity + u % rows, m);
  }
}

void launch_bucket_reduce(const DevTable* h_tab, uint32_t n_tables, const uint16_t* d_su, cudaStream_t s) {
  for (uint32_t t = 0; t < n_tables; ++t) {
    const DevTable& T = h_tab[t];
    if (T.su <= 1) continue;
    const mark_t* sub[3] = {T.sub[0], T.sub[1], T.sub[2]};
    mark_t* word[3] = {T.wmarks, T.amarks, T.rmarks};
    const uint32_t groups[3] = {T.n_groups, (uint32_t)__builtin_popcount(T.add_groups), T.n_groups};
    for (int k = 0; k < 3; ++k) {
      if (!sub[k] || !word[k] || !groups[k] || !T.sub_rows) continue;
      const uint64_t warps = (uint64_t)groups[k] * T.sub_rows * ((T.su + 1023) / 1024);
      const unsigned blocks = (unsigned)std::min<uint64_t>((warps + 7) / 8, 148 * 8);
      k_bucket_reduce<<<blocks, 256, 0, s>>>(sub[k], word[k], groups[k], T.sub_rows, T.capacity, T.su, d_su, t);
      note_launch();
    }
  }
}

// T per table: OPS batches (kcount == null): every txn may access every table (YCSB's one table:
// exact).  TPC-C: the sum of the per-procedure list lengths of the procedures that access the
// table (NewOrder: W D C I S + inserts into O NO OL; Payment: W D C H; OrderStatus: C O OL;
// Delivery: D NO O OL C; StockLevel: D O OL S).
__global__ void k_popularity(const uint32_t* kcount, uint32_t n_all, uint16_t* d_su, uint32_t* popular,
                             uint32_t n_tables) {
  constexpr uint32_t TPCC_ACCESS[5] = {0x1F7u, 0x00Fu, 0x064u, 0x076u, 0x162u};  // table bits per procedure
  const uint32_t t = threadIdx.x;
  uint32_t su = 1;
  if (t < n_tables) {
    const DevTable& T = c_tabs[t];
    if (T.su > 1 && T.sub_rows) {  // E = T / D > 1  <=>  T > D
      uint64_t cnt = n_all;
      if (kcount) {
        cnt = 0;
        for (int k = 0; k < 5; ++k)
          if ((TPCC_ACCESS[k] >> t) & 1u) cnt += kcount[k];
      }
      if (cnt > T.sub_rows) {
        const uint64_t e = (cnt + T.sub_rows - 1) / T.sub_rows;  // ceil(E); ceil(ceil(E)/32) == ceil(E/32)
        su = (uint32_t)((e + 31) / 32 * 32 < T.su ? (e + 31) / 32 * 32 : T.su);
      }
    }
    d_su[t] = (uint16_t)su;
  }
  const uint32_t m = __ballot_sync(0xffffffffu, su > 1);
  if (t == 0 && popular) *popular = m;
}

void launch_popularity(const DevTable* h_tab, uint32_t n_tables, const uint32_t* kcount, uint32_t n_all,
                       uint16_t* d_su, uint32_t* popular, cudaStream_t s) {
  bool any = false;
  for (uint32_t t = 0; t < n_tables; ++t) any |= h_tab[t].su > 1;
  if (!any) return;
  static_assert(MAXT <= 32, "one warp");
  k_popularity<<<1, 32, 0, s>>>(kcount, n_all, d_su, popular, n_tables);
  note_launch();
  upload_tables_common_su(d_su, s);
  upload_tables_ops_su(d_su, s);
  upload_tables_tpcc_su(d_su, s);
}

__global__ void k_scatter_col(long long* dst, uint32_t stride, const long long* src, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    dst[i * stride] = src[i];
}

void launch_scatter_col(long long* dst, uint32_t stride, const long long* src, uint64_t n, cudaStream_t s) {
  if (!n) return;
  k_scatter_col<<<148 * 16, 256, 0, s>>>(dst, stride, src, n);
  note_launch();
}

__global__ void k_build_index(uint32_t t, uint64_t row0, uint64_t n,
                              uint32_t* err) {
  const DevTable& T = c_tabs[t];
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t row = row0 + i;
    uint64_t key = T.rowkey[row];
    if (key == KEY_EMPTY) { atomicOr(err, ERR_EINVAL); continue; }
    IdxSlot* sl = idx_find_or_insert(T, key);
    if (!sl) { atomicOr(err, ERR_ECAPACITY); continue; }
    if (atomicCAS(&sl->row, ROW_NONE, (unsigned)row) != ROW_NONE) atomicOr(err, ERR_EINVAL);  // duplicate key
  }
}

// deferred index maintenance: index the valid rows [*from, n_rows) of table t
__global__ void k_build_index_tail(uint32_t t, const unsigned long long* from, uint32_t* err) {
  const DevTable& T = c_tabs[t];
  const uint64_t r0 = *from, r1 = *T.n_rows;
  for (uint64_t row = r0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; row < r1;
       row += (uint64_t)gridDim.x * blockDim.x) {
    if (!T.valid[row]) continue;
    IdxSlot* sl = idx_find_or_insert(T, T.rowkey[row]);
    if (!sl) { atomicOr(err, ERR_EINTERNAL); continue; }
    sl->row = (uint32_t)row;
  }
}

__global__ void k_note_rows(uint32_t t, unsigned long long* dst) { *dst = *c_tabs[t].n_rows; }

void launch_build_index_tail(uint32_t t, const unsigned long long* from, uint32_t* err, cudaStream_t s) {
  k_build_index_tail<<<148 * 8, 256, 0, s>>>(t, from, err);
  note_launch();
}

void launch_note_rows(uint32_t t, unsigned long long* dst, cudaStream_t s) {
  k_note_rows<<<1, 1, 0, s>>>(t, dst);
  note_launch();
}

void launch_build_index(uint32_t t, uint64_t row0, uint64_t n, uint32_t* err,
                        cudaStream_t s) {
  if (!n) return;
  uint64_t blocks = (n + 255) / 256;
  if (blocks > 148 * 64) blocks = 148 * 64;
  k_build_index<<<(unsigned)blocks, 256, 0, s>>>(t, row0, n, err);
  note_launch();
}

// ECAPACITY before anything mutates.  The partition's inserts take provisional rows
// n_rows + base + [0, total); base is this partition's offset in the batch reservation.
__global__ void k_capacity(uint32_t n_tables, const uint32_t* ins_tables, const uint32_t* total,
                           unsigned long long* base, unsigned long long* reserve, uint32_t* err) {
  capacity_body(n_tables, ins_tables, total, base, reserve, err);
}

void launch_capacity_check(uint32_t n_tables, const uint32_t* ins_tables, const uint32_t* total,
                           unsigned long long* base, unsigned long long* reserve, uint32_t* err, cudaStream_t s) {
  k_capacity<<<1, 1, 0, s>>>(n_tables, ins_tables, total, base, reserve, err);
  note_launch();
}

__global__ void k_advance(uint32_t n_tables, const unsigned long long* reserve, const uint32_t* err,
                          uint32_t* dense_live, const uint32_t* insdel) {
  if (*err) return;
  for (uint32_t t = 0; t < n_tables; ++t) *c_tabs[t].n_rows += reserve[t];
  *dense_live &= ~*insdel;  // a table that saw INSERT/DELETE is looked up by hash from now on
}

void launch_advance_cursor(uint32_t n_tables, const unsigned long long* reserve, const uint32_t* err,
                           uint32_t* dense_live, const uint32_t* insdel, cudaStream_t s) {
  k_advance<<<1, 1, 0, s>>>(n_tables, reserve, err, dense_live, insdel);
  note_launch();
}

}  // namespace ltpg
