// codec.cu — key codecs for the other key types and orders.
//
// The GPUSort (radix.cu) and the merges sort 64-bit unsigned "internal" keys ascending; the
// float64 ascending path fuses its order-preserving transform (A4) into the first and last radix
// pass.  Other orders and key types go through one encode pass before the sort and one decode
// pass after it, both HBM-bound elementwise kernels:
//
//   float64, descending   k = ~key64(u)                    (u = the float64 bits)
//   float32, ascending    k = key32(w)          (zero-extended: digits 4..7 are trivial and the
//   float32, descending   k = ~key32(w) & 2^32-1  radix plan skips them, so 4 LSD passes run)
//
// key32(w) = w >> 31 ? ~w : w | 2^31 is IEEE 754 totalOrder on binary32 as an unsigned compare
// (the 32-bit analogue of A4, P:253-264 / P:511-519 call 64-bit keys the worst case).  Every
// totalOrder class is a single bit pattern, so the descending result is the exact reverse of the
// ascending one and both are unique.
#include <cuda_runtime.h>

#include <cstdint>

#include "internal.h"

namespace hsort {
namespace {

__device__ __forceinline__ uint64_t key64(uint64_t u) {
  return u ^ ((uint64_t)((int64_t)u >> 63) | 0x8000000000000000ull);
}
__device__ __forceinline__ uint64_t unkey64(uint64_t k) {
  return k ^ ((uint64_t)((int64_t)(~k) >> 63) | 0x8000000000000000ull);
}
__device__ __forceinline__ uint32_t key32(uint32_t w) {
  return w ^ ((uint32_t)((int32_t)w >> 31) | 0x80000000u);
}
__device__ __forceinline__ uint32_t unkey32(uint32_t k) {
  return k ^ ((uint32_t)((int32_t)(~k) >> 31) | 0x80000000u);
}

// KT: 0 = float64, 1 = float32.  Grid-stride over 2 (f64) or 4 (f32) elements per step with
// 16-byte loads; the < 4-element tail is done by thread 0 of block 0.
template <int KT>
__global__ void k_encode(const void* __restrict__ in, uint64_t* __restrict__ out, uint64_t n,
                         int desc) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t t0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (KT == 0) {
    const uint64_t x = desc ? ~0ull : 0ull;
    const ulonglong2* src = (const ulonglong2*)in;
    ulonglong2* dst = (ulonglong2*)out;
    for (uint64_t i = t0; i < n / 2; i += stride) {
      ulonglong2 v = __ldcs(src + i);
      v.x = key64(v.x) ^ x;
      v.y = key64(v.y) ^ x;
      __stcs(dst + i, v);
    }
    if (t0 == 0 && (n & 1)) out[n - 1] = key64(((const uint64_t*)in)[n - 1]) ^ x;
  } else {
    const uint32_t x = desc ? 0xFFFFFFFFu : 0u;
    const uint4* src = (const uint4*)in;
    for (uint64_t i = t0; i < n / 4; i += stride) {
      const uint4 v = __ldcs(src + i);
      ulonglong2 a, b;
      a.x = key32(v.x) ^ x;
      a.y = key32(v.y) ^ x;
      b.x = key32(v.z) ^ x;
      b.y = key32(v.w) ^ x;
      __stcs((ulonglong2*)(out + 4 * i), a);
      __stcs((ulonglong2*)(out + 4 * i + 2), b);
    }
    if (t0 == 0)
      for (uint64_t i = n & ~3ull; i < n; ++i) out[i] = key32(((const uint32_t*)in)[i]) ^ x;
  }
}

template <int KT>
__global__ void k_decode(const uint64_t* __restrict__ in, void* __restrict__ out, uint64_t n,
                         int desc) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t t0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (KT == 0) {
    const uint64_t x = desc ? ~0ull : 0ull;
    const ulonglong2* src = (const ulonglong2*)in;
    ulonglong2* dst = (ulonglong2*)out;
    for (uint64_t i = t0; i < n / 2; i += stride) {
      ulonglong2 v = __ldcs(src + i);
      v.x = unkey64(v.x ^ x);
      v.y = unkey64(v.y ^ x);
      __stcs(dst + i, v);
    }
    if (t0 == 0 && (n & 1)) ((uint64_t*)out)[n - 1] = unkey64(in[n - 1] ^ x);
  } else {
    const uint32_t x = desc ? 0xFFFFFFFFu : 0u;
    uint4* dst = (uint4*)out;
    for (uint64_t i = t0; i < n / 4; i += stride) {
      const ulonglong2 a = __ldcs((const ulonglong2*)(in + 4 * i));
      const ulonglong2 b = __ldcs((const ulonglong2*)(in + 4 * i + 2));
      uint4 v;
      v.x = unkey32((uint32_t)a.x ^ x);
      v.y = unkey32((uint32_t)a.y ^ x);
      v.z = unkey32((uint32_t)b.x ^ x);
      v.w = unkey32((uint32_t)b.y ^ x);
      __stcs(dst + i, v);
    }
    if (t0 == 0)
      for (uint64_t i = n & ~3ull; i < n; ++i) ((uint32_t*)out)[i] = unkey32((uint32_t)in[i] ^ x);
  }
}

unsigned codec_grid(uint64_t work) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint64_t want = (work + 255) / 256;
  const uint64_t cap = (uint64_t)sms * 8;  // 8 x 256-thread CTAs per SM, grid-stride
  return (unsigned)(want < cap ? (want ? want : 1) : cap);
}

}  // namespace

cudaError_t key_encode(const void* in, uint64_t* out, uint64_t n, int key_type, bool desc,
                       cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  if ((((uintptr_t)in) | ((uintptr_t)out)) & 15) return cudaErrorMisalignedAddress;
  if (key_type == kKeyF64)
    k_encode<0><<<codec_grid(n / 2), 256, 0, st>>>(in, out, n, desc ? 1 : 0);
  else if (key_type == kKeyF32)
    k_encode<1><<<codec_grid(n / 4), 256, 0, st>>>(in, out, n, desc ? 1 : 0);
  else
    return cudaErrorInvalidValue;
  return launched();
}

cudaError_t key_decode(const uint64_t* in, void* out, uint64_t n, int key_type, bool desc,
                       cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  if ((((uintptr_t)in) | ((uintptr_t)out)) & 15) return cudaErrorMisalignedAddress;
  if (key_type == kKeyF64)
    k_decode<0><<<codec_grid(n / 2), 256, 0, st>>>(in, out, n, desc ? 1 : 0);
  else if (key_type == kKeyF32)
    k_decode<1><<<codec_grid(n / 4), 256, 0, st>>>(in, out, n, desc ? 1 : 0);
  else
    return cudaErrorInvalidValue;
  return launched();
}

}  // namespace hsort
