// transfer.cu -- the cold path's transfer encoding (the
// paper's bottleneck is the PCIe copy): ddq_load_column keeps, next to
// the raw pinned copy, a frame-of-reference BIT-packed copy (value - vmin in the
// bit length of the column's range, 1..32 bits, a little-endian bit stream) and a
// cold cache miss copies that and widens it on the device.  When fewer bytes, the
// stream holds ranks into a sorted dictionary of the column's distinct values, sent
// behind it (yyyymmdd dates: 2556 distinct days in 12 bits instead of a 17-bit
// range).  SSB lineorder at SF20 moves 18.4 bytes per row over the link with the
// range code (whole-byte packing, round 1: 21; raw: 56).
#include <cstdint>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "ops_internal.h"

namespace ddq {

namespace {

// thread i: value i = bits [i*b, i*b + b) of the little-endian packed stream (b <= 32,
// so it lies in two consecutive 32-bit words; the stream carries a padding word)
template <int W>
__global__ void unpack_bits_kernel(const uint32_t* __restrict__ packed, int bits, long long base, void* __restrict__ out,
                                   uint32_t n, const long long* __restrict__ dict) {
  const uint64_t mask = bits == 32 ? 0xFFFFFFFFull : ((1ull << bits) - 1);
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint64_t o = (uint64_t)i * (uint32_t)bits;
    const size_t wi = (size_t)(o >> 5);
    const uint64_t two = (uint64_t)__ldg(packed + wi) | ((uint64_t)__ldg(packed + wi + 1) << 32);
    const uint64_t code = (two >> (o & 31)) & mask;
    const long long v = dict ? __ldg(dict + code) : base + (long long)code;
    if (W == 4) reinterpret_cast<int32_t*>(out)[i] = (int32_t)v;
    else reinterpret_cast<long long*>(out)[i] = v;
  }
}

}  // namespace

size_t packed_bytes(int64_t n, int bits) { return ((size_t)n * (size_t)bits + 7) / 8 / 16 * 16 + 48; }

cudaError_t launch_unpack(const void* packed, int bits, int64_t base, void* out, int width, int64_t n, cudaStream_t st,
                          const void* dict) {
  if (n <= 0) return cudaSuccess;
  if (n > 0xFFFFFFFFll || (width != 4 && width != 8) || bits < 1 || bits > 32) return cudaErrorInvalidValue;
  int64_t grid = (n + 255) / 256;
  if (grid > (int64_t)num_sms() * 16) grid = (int64_t)num_sms() * 16;
  const uint32_t* p = reinterpret_cast<const uint32_t*>(packed);
  const long long* dv = reinterpret_cast<const long long*>(dict);
  if (width == 4) unpack_bits_kernel<4><<<(int)grid, 256, 0, st>>>(p, bits, base, out, (uint32_t)n, dv);
  else unpack_bits_kernel<8><<<(int)grid, 256, 0, st>>>(p, bits, base, out, (uint32_t)n, dv);
  return cudaGetLastError();
}

}  // namespace ddq
