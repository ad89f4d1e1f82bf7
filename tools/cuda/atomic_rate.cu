// Same-address global atomicAdd throughput (one atomic per warp, returned value used).
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(unsigned* c, unsigned* sink, int iters) {
  unsigned acc = 0;
  for (int i = 0; i < iters; i++) {
    unsigned v = 0;
    if ((threadIdx.x & 31) == 0) v = atomicAdd(c, 1u);
    acc += __shfl_sync(0xffffffffu, v, 0);
  }
  if (acc == 0xFFFFFFFFu) sink[0] = acc;
}
int main() {
  unsigned *c, *s;
  cudaMalloc(&c, 4);
  cudaMalloc(&s, 4);
  for (int warps_per_sm : {8, 16, 32}) {
    int grid = 148, block = warps_per_sm * 32, iters = 64;
    k<<<grid, block>>>(c, s, iters);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    k<<<grid, block>>>(c, s, iters);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    double n = (double)grid * warps_per_sm * iters;
    printf("warps/SM %d: %.0f atomics in %.1f us -> %.2f G atomics/s\n", warps_per_sm, n, ms * 1e3, n / ms / 1e6);
  }
  return 0;
}
