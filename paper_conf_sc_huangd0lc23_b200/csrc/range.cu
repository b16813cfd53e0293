// range.cu -- value-range reduction for REL error bounds (SURVEY 8(a) row
// a1; Eq 1: eb = lambda * r, r = max - min; R3, R4).
//
// HBM-bound: grid-stride 128-bit streaming loads (4 in flight per thread),
// per-thread max/min on ORDER-PRESERVING 32-bit keys (so NaN propagates and
// -0 < +0 like the bit order), warp shuffles, one smem pass, one atomicMax
// pair per CTA; the last CTA decodes the keys, writes (min, max) and resets
// the accumulators to their identity 0 (so the workspace needs no memset).
#include "internal.cuh"

#ifndef CUSZP_RANGE_UNROLL
#define CUSZP_RANGE_UNROLL 4
#endif

namespace cuszp {

namespace {

__device__ __forceinline__ uint32_t order_key(float f) {
  const uint32_t u = __float_as_uint(f);
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ float key_to_float(uint32_t k) {
  return __uint_as_float((k & 0x80000000u) ? (k & 0x7fffffffu) : ~k);
}

}  // namespace

__global__ void __launch_bounds__(256) range_kernel(RangeArgs a) {
  pdl_launch_dependents();   // the compression kernel may be scheduled as these CTAs retire
  uint32_t kmax = 0u;          // max key
  uint32_t kmin = 0xffffffffu; // min key
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t nthreads = uint64_t(gridDim.x) * blockDim.x;

  const bool aligned = (reinterpret_cast<uintptr_t>(a.in) & 15u) == 0;
  uint64_t done = 0;
  if (aligned) {
    const uint64_t n4 = a.n / 4;
    const float4* in4 = reinterpret_cast<const float4*>(a.in);
    constexpr int U = CUSZP_RANGE_UNROLL;
    uint64_t i = tid;
    for (; i + (U - 1) * nthreads < n4; i += U * nthreads) {
      float4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = ld_stream_f32x4(in4 + i + u * nthreads);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint32_t k0 = order_key(v[u].x), k1 = order_key(v[u].y);
        const uint32_t k2 = order_key(v[u].z), k3 = order_key(v[u].w);
        kmax = max(kmax, max(max(k0, k1), max(k2, k3)));
        kmin = min(kmin, min(min(k0, k1), min(k2, k3)));
      }
    }
    for (; i < n4; i += nthreads) {
      const float4 v = ld_stream_f32x4(in4 + i);
      const uint32_t k0 = order_key(v.x), k1 = order_key(v.y);
      const uint32_t k2 = order_key(v.z), k3 = order_key(v.w);
      kmax = max(kmax, max(max(k0, k1), max(k2, k3)));
      kmin = min(kmin, min(min(k0, k1), min(k2, k3)));
    }
    done = n4 * 4;
  }
  for (uint64_t i = done + tid; i < a.n; i += nthreads) {
    const uint32_t k = order_key(ld_stream_f32(a.in + i));
    kmax = max(kmax, k);
    kmin = min(kmin, k);
  }

  kmax = __reduce_max_sync(kFull, kmax);
  kmin = __reduce_min_sync(kFull, kmin);
  __shared__ uint32_t s_max[8], s_min[8];
  __shared__ int s_last;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (lane == 0) { s_max[warp] = kmax; s_min[warp] = kmin; }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < int(blockDim.x >> 5); ++w) { kmax = max(kmax, s_max[w]); kmin = min(kmin, s_min[w]); }
    atomicMax(&a.ws->range_max_key, kmax);
    atomicMax(&a.ws->range_min_key, ~kmin);
    __threadfence();
    s_last = (atomicAdd(&a.ws->range_exit, 1u) == gridDim.x - 1);
    if (s_last) {
      __threadfence();
      const uint32_t gmax = atomicExch(&a.ws->range_max_key, 0u);
      const uint32_t gmin = ~atomicExch(&a.ws->range_min_key, 0u);
      float mn = key_to_float(gmin), mx = key_to_float(gmax);
      if (isnan(mn) || isnan(mx)) mn = mx = __int_as_float(0x7fc00000);
      a.ws->minmax[0] = mn;
      a.ws->minmax[1] = mx;
      if (a.user_minmax) { a.user_minmax[0] = mn; a.user_minmax[1] = mx; }
      a.ws->range_exit = 0;
      __threadfence();
    }
  }
}

}  // namespace cuszp
