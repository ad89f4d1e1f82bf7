// Gather micro-benchmark: DRAM cost of reading one int32 / int64 per selected row
// of a 120M-row column at TID densities d (sorted TIDs), with different load
// flavours.  Answers: what DRAM granularity do sparse gathers pay on B200, and
// does a load qualifier change it?  (Run alone for times; under
// `ncu --metrics dram__bytes_read.sum` for bytes.)
#include <cstdint>
#include <cmath>
#include <cstdio>
#include <vector>
#include <cuda_runtime.h>

template <int kMode, typename T>
__global__ void gather(const T* __restrict__ col, const int32_t* __restrict__ tids, uint32_t n, T* out) {
  T acc = 0;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const T* p = col + tids[i];
    T v;
    if (kMode == 0) {
      v = __ldg(p);
    } else if (kMode == 1) {
      v = *p;  // ld.global (L1-allocating)
    } else if (kMode == 2) {
      v = __ldcg(p);  // ld.global.cg (L2 only)
    } else if (kMode == 3) {
      v = __ldcs(p);  // ld.global.cs (evict-first)
    } else {
      if (sizeof(T) == 8) {
        unsigned long long x;
        asm volatile("ld.global.nc.L1::no_allocate.L2::64B.u64 %0, [%1];" : "=l"(x) : "l"(p));
        v = (T)x;
      } else {
        unsigned x;
        asm volatile("ld.global.nc.L1::no_allocate.L2::64B.u32 %0, [%1];" : "=r"(x) : "l"(p));
        v = (T)x;
      }
    }
    acc += v;
  }
  if (acc == (T)0x7fffffff) out[0] = acc;
}

static uint64_t mix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

template <int kMode, typename T>
float run(const T* col, const int32_t* tids, uint32_t n, T* out) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  gather<kMode, T><<<148 * 8, 256>>>(col, tids, n, out);
  cudaEventRecord(a);
  for (int r = 0; r < 5; r++) gather<kMode, T><<<148 * 8, 256>>>(col, tids, n, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  return ms / 5;
}

int main() {
  const uint32_t N = 120000000u;
  int64_t* c64;
  int32_t* c32;
  int32_t* tids;
  int64_t* o64;
  int32_t* o32;
  cudaMalloc(&c64, (size_t)N * 8);
  cudaMalloc(&c32, (size_t)N * 4);
  cudaMalloc(&tids, (size_t)N * 4);
  cudaMalloc(&o64, 64);
  cudaMalloc(&o32, 64);
  cudaMemset(c64, 1, (size_t)N * 8);
  cudaMemset(c32, 1, (size_t)N * 4);
  for (double d : {0.02, 0.04, 0.14, 0.2}) {
    std::vector<int32_t> h;
    h.reserve((size_t)(N * d * 1.1));
    for (uint32_t i = 0; i < N; i++)
      if ((double)(mix(i) >> 11) * (1.0 / 9007199254740992.0) < d) h.push_back((int32_t)i);
    cudaMemcpy(tids, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    const uint32_t n = (uint32_t)h.size();
    const double s32 = (double)N * 4 * (1 - std::pow(1 - d, 8.0)) / 1e6;   // 32 B sectors, int32
    const double s64 = (double)N * 8 * (1 - std::pow(1 - d, 4.0)) / 1e6;   // 32 B sectors, int64
    printf("density %.2f: %u TIDs; 32B-sector model: int32 %.0f MB, int64 %.0f MB\n", d, n, s32, s64);
    const char* names[5] = {"ldg.nc", "ld.global", "ld.cg", "ld.cs", "nc.L2::64B"};
    float t64[5] = {run<0>(c64, tids, n, o64), run<1>(c64, tids, n, o64), run<2>(c64, tids, n, o64),
                    run<3>(c64, tids, n, o64), run<4>(c64, tids, n, o64)};
    float t32[5] = {run<0>(c32, tids, n, o32), run<1>(c32, tids, n, o32), run<2>(c32, tids, n, o32),
                    run<3>(c32, tids, n, o32), run<4>(c32, tids, n, o32)};
    for (int k = 0; k < 5; k++)
      printf("  %-11s int64 %7.1f us (%6.0f GB/s of model)   int32 %7.1f us (%6.0f GB/s of model)\n", names[k],
             t64[k] * 1e3, s64 / t64[k], t32[k] * 1e3, s32 / t32[k]);
  }
  return 0;
}
