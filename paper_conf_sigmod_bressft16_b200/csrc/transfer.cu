// transfer.cu -- the cold path's transfer encoding (the
// paper's bottleneck is the PCIe copy): ddq_load_column keeps, next to
// the raw pinned copy, a frame-of-reference byte-packed copy (value - vmin in the
// fewest whole bytes, 1..4, little endian) and a cold cache miss copies that and
// widens it on the device.  SSB lineorder at SF20 moves 21 instead of 56 bytes per
// row over the link.
//
// Widening: thread i handles elements 4i..4i+3 = TW 32-bit words of the packed
// stream (4 * TW bytes, word-aligned), writes 4 outputs with vector stores.
#include <cstdint>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "ops_internal.h"

namespace ddq {

namespace {

template <int TW, int W>
__global__ void unpack_kernel(const uint32_t* __restrict__ packed, long long base, void* __restrict__ out,
                              uint32_t n) {
  const uint32_t groups = (n + 3) / 4;
  for (uint32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < groups; g += gridDim.x * blockDim.x) {
    uint32_t w[TW + 1];
#pragma unroll
    for (int k = 0; k < TW; k++) w[k] = __ldcs(packed + (size_t)g * TW + k);
    w[TW] = 0;
    long long v[4];
#pragma unroll
    for (int i = 0; i < 4; i++) {
      constexpr uint64_t mask = TW == 4 ? 0xFFFFFFFFull : ((1ull << (8 * TW)) - 1);
      const int bit = i * TW * 8, wi = bit >> 5, sh = bit & 31;
      const uint64_t two = (uint64_t)w[wi] | ((uint64_t)w[wi + 1] << 32);
      v[i] = base + (long long)((two >> sh) & mask);
    }
    const uint32_t e0 = g * 4;
    if (e0 + 4 <= n) {
      if (W == 4) {
        reinterpret_cast<int4*>(out)[g] = make_int4((int)v[0], (int)v[1], (int)v[2], (int)v[3]);
      } else {
        longlong2* o = reinterpret_cast<longlong2*>(out) + (size_t)g * 2;
        o[0] = make_longlong2(v[0], v[1]);
        o[1] = make_longlong2(v[2], v[3]);
      }
    } else {
      for (int i = 0; i < 4 && e0 + i < n; i++) {
        if (W == 4) reinterpret_cast<int32_t*>(out)[e0 + i] = (int32_t)v[i];
        else reinterpret_cast<long long*>(out)[e0 + i] = v[i];
      }
    }
  }
}

template <int TW>
void launch_tw(const void* packed, long long base, void* out, int width, uint32_t n, int grid, cudaStream_t st) {
  const uint32_t* p = reinterpret_cast<const uint32_t*>(packed);
  if (width == 4) unpack_kernel<TW, 4><<<grid, 256, 0, st>>>(p, base, out, n);
  else unpack_kernel<TW, 8><<<grid, 256, 0, st>>>(p, base, out, n);
}

}  // namespace

size_t packed_bytes(int64_t n, int tw) { return ((size_t)n * tw + 15) / 16 * 16 + 32; }

cudaError_t launch_unpack(const void* packed, int tw, int64_t base, void* out, int width, int64_t n, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  if (n > 0xFFFFFFFFll || (width != 4 && width != 8) || tw < 1 || tw > 4) return cudaErrorInvalidValue;
  int64_t grid = ((n + 3) / 4 + 255) / 256;
  if (grid > (int64_t)num_sms() * 16) grid = (int64_t)num_sms() * 16;
  switch (tw) {
    case 1: launch_tw<1>(packed, base, out, width, (uint32_t)n, (int)grid, st); break;
    case 2: launch_tw<2>(packed, base, out, width, (uint32_t)n, (int)grid, st); break;
    case 3: launch_tw<3>(packed, base, out, width, (uint32_t)n, (int)grid, st); break;
    default: launch_tw<4>(packed, base, out, width, (uint32_t)n, (int)grid, st); break;
  }
  return cudaGetLastError();
}

}  // namespace ddq
