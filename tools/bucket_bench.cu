// Table VII / VIII microbenchmark (NEXT-3, §V-C, §VI-D).
//
// N = Grid x Block threads (1024x1024 and 512x512, the paper's shapes) record their TID in a
// conflict table of H units (H = 1, 32, 512: "hash table" size, i.e. how many distinct rows the
// threads contend on; thread t -> unit t mod H), then read it back (conflict check: the unit's
// minimum TID vs the thread's own).  Each cell reports the paper's triplet
//   (mark + read, mark only, read only) in microseconds
// for the standard-sized bucket (s_u = 1: one mark word per unit, atomicMin) and the large-sized
// bucket (s_u = 32: sub-slot TID mod s_u; the read folds each bucket to its minimum once,
// P:225, then every thread checks one word),
// plus the two B200 variants the library uses instead: the read-before-atomicMin filter (the
// default, ltpg_internal.cuh mark_min) and warp aggregation (__match_any_sync + __reduce_min_sync,
// one atomic per distinct unit in the warp).  The mark words are the library's own epoch-tagged
// 32-bit format and mark_min / mark_rank functions.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include tools/bucket_bench.cu
#include <algorithm>
#include <cstdio>
#include <vector>

#include "../paper_conf_icde_wei0l0lzj024_b200/csrc/ltpg_internal.cuh"

using namespace ltpg;

enum { V_STD = 0, V_LARGE = 1, V_FILTER = 2, V_WARPAGG = 3 };
static const char* VNAME[] = {"s_u=1 (standard, atomicMin)", "s_u=32 (large bucket)",
                              "s_u=1 + read-before-atomicMin filter (library default)",
                              "s_u=1 + warp aggregation (match_any + reduce_min)"};
constexpr uint32_t EPOCH = 7;

template <int V>
__global__ void k_mark(mark_t* tab, uint32_t H, uint32_t su) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;  // TID (rank)
  const uint32_t u = t % H;
  const mark_t tag = epoch_tag(EPOCH) | t;
  if (V == V_STD) mark_min(tab + u, tag, false);
  if (V == V_FILTER) mark_min(tab + u, tag, true);
  if (V == V_LARGE) mark_min(tab + (uint64_t)u * su + t % su, tag, false);
  if (V == V_WARPAGG) {
    const uint32_t peers = __match_any_sync(0xffffffffu, u);
    const mark_t m = __reduce_min_sync(peers, tag);
    if ((threadIdx.x & 31) == (uint32_t)(__ffs(peers) - 1)) atomicMin(tab + u, m);
  }
}

// large buckets: the bucket's minimum ("reads out all the TIDs in the hash bucket and selects
// ... the smallest") folded once per bucket into its unit word -- one warp per bucket, as
// the library's k_bucket_reduce does -- before the per-thread check
__global__ void k_fold(const mark_t* sub, mark_t* word, uint32_t H, uint32_t su) {
  const uint32_t u = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (u >= H) return;
  mark_t m = 0xFFFFFFFFu;
  for (uint32_t j = lane; j < su; j += 32) m = min(m, __ldcg(sub + (uint64_t)u * su + j));
  m = __reduce_min_sync(0xffffffffu, m);
  if (lane == 0) word[u] = m;
}

// conflict check: the unit's minimum TID vs the thread's own
__global__ void k_read(const mark_t* tab, uint32_t H, uint32_t* out) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t m = mark_rank(__ldcg(tab + t % H), EPOCH);
  if (m < t) atomicAdd(out, 1u);  // a WAW conflict for everyone but the smallest TID
}

int main() {
  const uint32_t shapes[2][2] = {{1024, 1024}, {512, 512}};
  const uint32_t Hs[3] = {1, 32, 512};
  mark_t *tab, *word;
  uint32_t* out;
  cudaMalloc(&tab, 512 * 32 * sizeof(mark_t));
  cudaMalloc(&word, 512 * sizeof(mark_t));
  cudaMalloc(&out, sizeof(uint32_t));
  cudaEvent_t e[3];
  for (auto& x : e) cudaEventCreate(&x);
  std::printf("{\"table\": \"VII\", \"unit\": \"us\", \"rows\": [\n");
  bool first = true;
  for (auto& sh : shapes) {
    const uint32_t grid = sh[0], block = sh[1], N = grid * block;
    for (uint32_t H : Hs) {
      for (int v = 0; v < 4; ++v) {
        const uint32_t su = v == V_LARGE ? 32 : 1;
        std::vector<float> mk, rd;
        for (int rep = 0; rep < 25; ++rep) {
          cudaMemset(tab, 0xFF, 512 * 32 * sizeof(mark_t));
          cudaMemset(out, 0, sizeof(uint32_t));
          cudaDeviceSynchronize();
          cudaEventRecord(e[0]);
          switch (v) {
            case V_STD: k_mark<V_STD><<<grid, block>>>(tab, H, su); break;
            case V_LARGE: k_mark<V_LARGE><<<grid, block>>>(tab, H, su); break;
            case V_FILTER: k_mark<V_FILTER><<<grid, block>>>(tab, H, su); break;
            default: k_mark<V_WARPAGG><<<grid, block>>>(tab, H, su); break;
          }
          cudaEventRecord(e[1]);
          if (v == V_LARGE) {
            k_fold<<<(H * 32 + 255) / 256, 256>>>(tab, word, H, su);
            k_read<<<grid, block>>>(word, H, out);
          } else {
            k_read<<<grid, block>>>(tab, H, out);
          }
          cudaEventRecord(e[2]);
          cudaEventSynchronize(e[2]);
          float a, b;
          cudaEventElapsedTime(&a, e[0], e[1]);
          cudaEventElapsedTime(&b, e[1], e[2]);
          if (rep >= 5) mk.push_back(1000 * a), rd.push_back(1000 * b);
        }
        uint32_t conflicts = 0;
        cudaMemcpy(&conflicts, out, sizeof(conflicts), cudaMemcpyDeviceToHost);
        std::sort(mk.begin(), mk.end());
        std::sort(rd.begin(), rd.end());
        const float m = mk[mk.size() / 2], r = rd[rd.size() / 2];
        std::printf("%s {\"grid\": %u, \"block\": %u, \"hash_table\": %u, \"variant\": \"%s\", \"s_u\": %u, "
                    "\"mark_read\": %.1f, \"mark\": %.1f, \"read\": %.1f, \"conflicts\": %u, \"expected\": %u}\n",
                    first ? " " : ",", grid, block, H, VNAME[v], su, m + r, m, r, conflicts, N - H);
        first = false;
      }
    }
  }
  std::printf("]}\n");
  const cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) {
    std::fprintf(stderr, "CUDA error: %s\n", cudaGetErrorString(err));
    return 1;
  }
  return 0;
}
