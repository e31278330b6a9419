// Helpers of the single-launch (cooperative) small-batch kernels: k_ops_small (k_ops.cu) and
// k_tpcc_small (k_tpcc.cu).  Stages are separated by grid-wide barriers; the grid's a8 block
// writes the commit bitmask, the counts and the abort list; the last block to finish publishes
// the slot's result words into mapped host memory.
#pragma once
#include "ltpg_internal.cuh"

namespace ltpg {

struct SmallOut {
  unsigned long long* reserve;  // [MAXT] append reservations (cleared here)
  BatchVars* vars;              // written here from (epoch, clock) or the slot's mapped host copy
  const volatile BatchVars* host;
  uint32_t epoch;
  long long clock;
  uint32_t* commit_bits;        // a8 outputs (as k_finalize_compact)
  uint32_t* dsmall;             // the slot's words: [0] err (written iff write0) [8..10] counts [16] n
  uint32_t* abort_out;
  uint32_t* n_out2;             // or null
  volatile uint32_t* host_small;  // the slot's mapped host words: [0..16] of dsmall, err ORed into [0]
  bool write0;
  uint32_t* bar;                // grid-barrier counter: zero at launch, on its own 128-byte line (the
                                // spinning blocks' polls stay off the error / count words), cleared
                                // by the last block
};

// a8 for n txns in one block: 32 txns per thread-word, block-wide scan of the conflict counts
// per 256-word round (carried), abort list in ascending rank order.  st_of(r) = txn r's status.
template <class St>
__device__ __forceinline__ void finalize_block(uint32_t n, const SmallOut& o, St st_of) {
  __shared__ uint32_t fw[8], fcarry, fred[3];
  const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (threadIdx.x == 0) fcarry = 0;
  if (threadIdx.x < 3) fred[threadIdx.x] = 0;
  __syncthreads();
  const uint32_t nw = (n + 31) / 32;
  for (uint32_t base = 0; base < nw; base += blockDim.x) {
    const uint32_t w = base + threadIdx.x;
    uint32_t cm = 0, am = 0, nu = 0;
    if (w < nw) {
      const uint32_t r0 = w * 32, m = min(32u, n - r0);
#pragma unroll 8
      for (uint32_t j = 0; j < m; ++j) {
        const uint8_t st = st_of(r0 + j);
        cm |= (st == LTPG_ST_COMMIT ? 1u : 0u) << j;
        am |= (st == LTPG_ST_CONFLICT ? 1u : 0u) << j;
        nu += st == LTPG_ST_USER_ABORT;
      }
      o.commit_bits[w] = cm;
    }
    const uint32_t na = __popc(am);
    uint32_t x = na;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, d);
      if (lane >= (uint32_t)d) x += y;
    }
    const uint32_t nbw = __reduce_add_sync(0xffffffffu, __popc(cm)), nuw = __reduce_add_sync(0xffffffffu, nu);
    if (lane == 31) fw[wid] = x;
    if (lane == 0) {
      atomicAdd(fred + 0, nbw);
      atomicAdd(fred + 2, nuw);
    }
    __syncthreads();
    uint32_t before = fcarry, round = 0;
#pragma unroll
    for (uint32_t q = 0; q < 8; ++q) {
      if (q < wid) before += fw[q];
      round += fw[q];
    }
    uint32_t pos = before + x - na;
    for (uint32_t m = am; m; m &= m - 1) o.abort_out[pos++] = w * 32 + (__ffs(m) - 1);
    __syncthreads();
    if (threadIdx.x == 0) fcarry += round;
  }
  __syncthreads();
  if (threadIdx.x < 17) {  // the slot's result words (the host memset of them is skipped)
    const uint32_t t = threadIdx.x;
    const uint32_t v = t == 8 ? fred[0] : t == 9 ? fcarry : t == 10 ? fred[2] : t == 16 ? fcarry : 0u;
    if (t || o.write0) o.dsmall[t] = v;
  }
  if (threadIdx.x == 0 && o.n_out2) *o.n_out2 = fcarry;
}

__device__ __forceinline__ void prefetch_l2(const void* p) { asm volatile("prefetch.global.L2 [%0];" ::"l"(p)); }

// Grid-wide barrier of a co-resident grid on a counter that is zero at launch: wait until
// `target` block arrivals were counted (one release-add per block, acquire polling by thread 0).
// About half the cost of cg::grid_group::sync on B200 (tools/launchcost.cu).  Barrier k of a
// grid where every block arrives at every barrier waits for k * gridDim.x arrivals.
__device__ __forceinline__ void grid_barrier_to(uint32_t* ctr, uint32_t target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr) : "memory");
    uint32_t v;
    do {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
    } while (v < target);
  }
  __syncthreads();
}
__device__ __forceinline__ void grid_barrier(uint32_t* ctr, uint32_t k) { grid_barrier_to(ctr, k * gridDim.x); }


}  // namespace ltpg
