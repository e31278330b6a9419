// Random-access ceiling of B200 HBM3e for the access shapes of the LTPG hot path:
// independent random 8-byte reads, random 8-byte atomicMin (mark RMW), and random
// 64-byte reads, over a 2 GiB array (>> 126 MB L2).  Reports accesses/s and the DRAM
// bytes they imply at 64 B per access (the B200 DRAM fetch granularity for a random miss).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o randbw tools/randbw.cu && ./randbw
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return x;
}

__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ unsigned long long ld_l2_64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.global.cg.L2::64B.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}

// 0: 8 B read (ld.cg), 1: 8 B atomicMin, 2: 64 B read (8 lanes x 8 B), 3: ld.global.nc,
// 4: plain ld, 5: ld.relaxed.gpu, 6: ld.cg.L2::64B
template <int MODE>
__global__ void k_rand(unsigned long long* a, uint64_t n, uint32_t iters, unsigned long long* sink) {
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  unsigned long long acc = 0;
  for (uint32_t i = 0; i < iters; ++i) {
    if (MODE == 2) {
      const uint64_t line = mix((tid >> 3) * 1315423911ull + i) & (n / 8 - 1);  // n is a power of two
      acc += __ldcg(a + line * 8 + (tid & 7));
    } else {
      const uint64_t j = mix(tid * 2654435761ull + i) & (n - 1);
      if (MODE == 0) acc += __ldcg(a + j);
      else if (MODE == 1) atomicMin(a + j, (unsigned long long)(tid + i));
      else if (MODE == 3) acc += __ldg(a + j);
      else if (MODE == 4) acc += a[j];
      else if (MODE == 5) acc += ld_relaxed(a + j);
      else acc += ld_l2_64(a + j);
    }
  }
  if (acc == 0x1234567) *sink = acc;
}

int main() {
  const uint64_t n = (2ull << 30) / 8;
  unsigned long long *a, *sink;
  cudaMalloc(&a, n * 8);
  cudaMalloc(&sink, 8);
  cudaMemset(a, 0x7F, n * 8);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const char* names[7] = {"random 8B ld.cg", "random 8B atomicMin", "random 64B read", "random 8B ld.nc",
                          "random 8B ld", "random 8B ld.relaxed", "random 8B ld.cg.L2::64B"};
  for (int mode = 0; mode < 7; ++mode)
    for (int bps : {8, 32}) {
      const int blocks = 148 * bps, threads = 256;
      const uint32_t iters = 64;
      float best = 1e30f;
      for (int rep = 0; rep < 4; ++rep) {
        cudaEventRecord(e0);
        if (mode == 0) k_rand<0><<<blocks, threads>>>(a, n, iters, sink);
        if (mode == 1) k_rand<1><<<blocks, threads>>>(a, n, iters, sink);
        if (mode == 2) k_rand<2><<<blocks, threads>>>(a, n, iters, sink);
        if (mode == 3) k_rand<3><<<blocks, threads>>>(a, n, iters, sink);
        if (mode == 4) k_rand<4><<<blocks, threads>>>(a, n, iters, sink);
        if (mode == 5) k_rand<5><<<blocks, threads>>>(a, n, iters, sink);
        if (mode == 6) k_rand<6><<<blocks, threads>>>(a, n, iters, sink);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep && ms < best) best = ms;
      }
      const double acc = (double)blocks * threads * iters / (mode == 2 ? 8 : 1);
      printf("%-22s blocks/SM %2d: %7.3f ms  %8.2f G accesses/s  %7.1f GB/s at 64 B/access\n", names[mode], bps,
             best, acc / best / 1e6, acc * 64 / best / 1e6);
    }
  printf("err: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
