// GPU-timeline cost of a plain vs a cooperative launch (17 x 256 threads), empty and with 4
// grid-wide barriers, N back to back between two timing events, after a host head start.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tools/launchcost tools/launchcost.cu
#include <cooperative_groups.h>
#include <cstdio>
namespace cg = cooperative_groups;

__global__ void k_empty(int* p) {
  if (p && threadIdx.x == 1023) *p = 1;
}
__global__ void k_sync(int* p, int nsync) {
  cg::grid_group g = cg::this_grid();
  for (int i = 0; i < nsync; ++i) g.sync();
  if (p && threadIdx.x == 1023) *p = 1;
}
__device__ __forceinline__ void gbar(unsigned* ctr, unsigned target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr) : "memory");
    unsigned v;
    do {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
    } while (v < target);
  }
  __syncthreads();
}
__global__ void k_mybar(unsigned* ctr, int nsync) {
  for (int i = 0; i < nsync; ++i) gbar(ctr, (i + 1) * gridDim.x);
  __syncthreads();
  if (threadIdx.x == 0) {  // last one out resets
    unsigned v = atomicAdd(ctr + 1, 1u);
    if (v == gridDim.x - 1) { ctr[0] = 0; ctr[1] = 0; }
  }
}
__global__ void k_spin(long long ns) {
  long long t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > ns) break;
  }
}

int main() {
  cudaStream_t s;
  cudaStreamCreate(&s);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int N = 50, G = 17;
  unsigned* ctr;
  cudaMalloc(&ctr, 8);
  cudaMemset(ctr, 0, 8);
  for (int mode = 0; mode < 6; ++mode) {
    float best = 1e9;
    for (int rep = 0; rep < 5; ++rep) {
      k_spin<<<1, 1, 0, s>>>(300000);  // 0.3 ms head start for the host
      cudaEventRecord(a, s);
      for (int i = 0; i < N; ++i) {
        int* np = nullptr;
        int ns = mode == 3 ? 1 : 4;
        void* args[] = {&np, &ns};
        if (mode == 0) k_empty<<<G, 256, 0, s>>>(nullptr);
        if (mode == 1) cudaLaunchCooperativeKernel((const void*)k_empty, dim3(G), dim3(256), args, 0, s);
        if (mode >= 2 && mode <= 3) cudaLaunchCooperativeKernel((const void*)k_sync, dim3(G), dim3(256), args, 0, s);
        if (mode == 4) k_empty<<<1, 32, 0, s>>>(nullptr);
        if (mode == 5) k_mybar<<<G, 256, 0, s>>>(ctr, 4);
      }
      cudaEventRecord(b, s);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      best = ms < best ? ms : best;
    }
    const char* name[] = {"plain 17x256", "cooperative 17x256 empty", "cooperative 17x256 4 grid.sync",
                          "cooperative 17x256 1 grid.sync", "plain 1x32",
                          "plain 17x256 4 release/acquire barriers"};
    printf("%-34s %.2f us per launch\n", name[mode], best * 1000.0f / N);
  }
  return 0;
}
