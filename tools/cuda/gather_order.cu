// Gather micro-benchmark, part 2: does the ORDER of a TID list change what a sparse
// int64 gather costs on B200?  Orders: sorted, runs of R sorted TIDs in random run
// order (what a compaction ring's block flushes produce), fully shuffled.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gather_order tools/cuda/gather_order.cu
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>
#include <cuda_runtime.h>

__global__ void gather(const long long* __restrict__ col, const int32_t* __restrict__ tids, uint32_t n,
                       long long* out) {
  long long acc = 0;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    long long v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::64B.s64 %0, [%1];" : "=l"(v) : "l"(col + tids[i]));
    acc += v;
  }
  if (acc == 0x7fffffff) out[0] = acc;
}

static uint64_t mix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

int main() {
  const uint32_t N = 120000000u;
  long long* col;
  int32_t* tids;
  long long* o;
  cudaMalloc(&col, (size_t)N * 8);
  cudaMalloc(&tids, (size_t)N * 4);
  cudaMalloc(&o, 64);
  cudaMemset(col, 1, (size_t)N * 8);
  std::mt19937_64 rng(7);
  for (double d : {0.016, 0.04, 0.2}) {
    std::vector<int32_t> h;
    for (uint32_t i = 0; i < N; i++)
      if ((double)(mix(i) >> 11) * (1.0 / 9007199254740992.0) < d) h.push_back((int32_t)i);
    const uint32_t n = (uint32_t)h.size();
    for (int R : {0, 1024, 128, 16, 1}) {  // 0: sorted; R: runs of R shuffled
      std::vector<int32_t> g = h;
      if (R > 0) {
        std::vector<uint32_t> runs((n + R - 1) / R);
        for (uint32_t r = 0; r < runs.size(); r++) runs[r] = r;
        std::shuffle(runs.begin(), runs.end(), rng);
        size_t k = 0;
        for (uint32_t r : runs)
          for (uint32_t i = r * R; i < std::min<uint32_t>(n, (r + 1) * R); i++) g[k++] = h[i];
      }
      cudaMemcpy(tids, g.data(), (size_t)n * 4, cudaMemcpyHostToDevice);
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      gather<<<148 * 8, 256>>>(col, tids, n, o);
      cudaEventRecord(a);
      for (int r = 0; r < 5; r++) gather<<<148 * 8, 256>>>(col, tids, n, o);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      ms /= 5;
      printf("density %.3f  %9u TIDs  order %-10s %7.1f us  %6.1f G gathers/s\n", d, n,
             R == 0 ? "sorted" : (R == 1 ? "shuffled" : (std::string("runs ") + std::to_string(R)).c_str()),
             ms * 1e3, n / ms / 1e6);
    }
  }
  return 0;
}
