// small_l.cu -- DIAGNOSTICS ONLY (built with -DCUSZP_SMALL_L_3PASS): the
// round-1 three-launch path for block lengths L in {8, 16}, kept as the A/B
// baseline of the one-pass kernels (compress.cu / decompress.cu, SL = 8 / 16,
// DESIGN 9.4).  The production library does not contain these kernels.
//
// One thread per L-block, tiles of 4096 elements:
//   compress:   sizes (quantise, Lorenzo, F, tile byte sums)  ->
//               tile scan + header (one CTA)                   ->
//               write (re-quantise, CTA scan of block bytes, sign map + planes)
//   decompress: sizes (F -> tile byte sums) -> tile scan + header check ->
//               decode (CTA scan, planes -> |l|, signs, prefix sum, r * 2eb)
//
// Status words: each tile's byte sum / exclusive prefix is stored < 2^40,
// so its epoch field is 0 and the look-back of the persistent kernels
// (epochs >= 1) never takes it for a published word.
#include "internal.cuh"

#ifdef CUSZP_SMALL_L_3PASS

namespace cuszp {
namespace {

constexpr int kSThreads = 256;
constexpr int kSTileElems = 4096;
constexpr int kScanThreads = 1024;

// eb_abs (Eq 1): ABS -> delta; REL -> lambda * (max - min) over the pairs (R3)
__device__ __forceinline__ float resolve_eb(const CompressArgs& a) {
  float eb = a.eb_in;
  if (a.mode == CUSZP_REL && a.n_pairs == 0) return 0.0f;   // R11
  if (a.mode == CUSZP_REL) {
    float mn = a.minmax[0], mx = a.minmax[1];
    bool nan = isnan(mn) || isnan(mx);
    for (int p = 1; p < a.n_pairs; ++p) {
      const float lo = a.minmax[2 * p], hi = a.minmax[2 * p + 1];
      nan |= isnan(lo) || isnan(hi);
      if (lo < mn) mn = lo;
      if (hi > mx) mx = hi;
    }
    eb = __fmul_rn(a.eb_in, __fsub_rn(mx, mn));
    if (nan) eb = __int_as_float(0x7fc00000);
  }
  return eb;
}

__device__ __forceinline__ bool eb_usable(float eb) {
  return (eb >= kFltMin) && isfinite(__fadd_rn(eb, eb));
}

// R2: r0 = nearest integer (ties to even) to the exact product d * recip,
// guard |r0| < 2^22 (R5), then the one-step correction that makes
// |d - r * 2eb| <= eb.  fma(d, recip, 1.5*2^23) rounds the exact product to
// an integer in ONE rounding while |d * recip| < 2^22, and every product at
// or beyond that fails the guard either way (DESIGN 8, the fast kernels'
// sequence).  Returns false when the guard fails (NaN and Inf included).
__device__ __forceinline__ bool quantize(float d, float eb, float two_eb, float recip, int32_t& r) {
  const float r0 = __fsub_rn(__fmaf_rn(d, recip, kRoundMagic), kRoundMagic);
  if (!(fabsf(r0) < kGuard)) { r = 0; return false; }
  const float res = __fmaf_rn(-r0, two_eb, d);
  r = int32_t(r0) + (res > eb ? 1 : 0) - (res < -eb ? 1 : 0);
  return true;
}

// One L-block: Lorenzo residuals l_i = r_i - r_{i-1} (r_{-1} = 0),
// returns F = bit length of max |l|; *bad on a guard failure.
// The L values of block k (zero pad beyond n, R8); whole blocks as float4.
template <int L>
__device__ __forceinline__ void block_load(const float* in, uint64_t n, uint64_t k, float* v) {
  if ((k + 1) * L <= n) {                                  // in is 16-byte aligned (ABI)
    const float4* p = reinterpret_cast<const float4*>(in + k * L);
#pragma unroll
    for (int q = 0; q < L / 4; ++q) {
      const float4 f = p[q];
      v[4 * q] = f.x; v[4 * q + 1] = f.y; v[4 * q + 2] = f.z; v[4 * q + 3] = f.w;
    }
  } else {
#pragma unroll
    for (int i = 0; i < L; ++i) v[i] = k * L + uint64_t(i) < n ? in[k * L + i] : 0.0f;
  }
}

// One L-block: Lorenzo residuals l_i = r_i - r_{i-1} (r_{-1} = 0),
// returns F = bit length of max |l|; *bad on a guard failure.
template <int L>
__device__ __forceinline__ int block_encode(const float* v, float eb, float two_eb, float recip, uint32_t* mag,
                                            uint32_t& sign, bool& bad) {
  int32_t prev = 0;
  uint32_t mx = 0;
  sign = 0;
#pragma unroll
  for (int i = 0; i < L; ++i) {
    int32_t r = 0;
    if (!quantize(v[i], eb, two_eb, recip, r)) bad = true;
    const int32_t l = r - prev;
    prev = r;
    if (l < 0) sign |= 1u << i;
    mag[i] = l < 0 ? uint32_t(-int64_t(l)) : uint32_t(l);
    mx = max(mx, mag[i]);
  }
  return mx == 0 ? 0 : 32 - __clz(int(mx));
}

// Exclusive CTA scan of one u32 per thread; *total = the CTA sum.
__device__ __forceinline__ uint32_t cta_excl_scan(uint32_t v, uint32_t* total) {
  __shared__ uint32_t s_warp[kSThreads / 32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_warp[warp] = x;
  __syncthreads();
  uint32_t base = 0, sum = 0;
#pragma unroll
  for (int w = 0; w < kSThreads / 32; ++w) {
    const uint32_t s = s_warp[w];
    if (w < warp) base += s;
    sum += s;
  }
  __syncthreads();
  *total = sum;
  return base + x - v;
}

// 8x8 bit-matrix transpose: bit p of byte i -> bit i of byte p.  Moves eight
// planes of eight elements at once (the block bit-shuffle, and its
// inverse) instead of one bit per instruction.
__device__ __forceinline__ uint64_t transpose8(uint64_t x) {
  uint64_t t;
  t = (x ^ (x >> 7)) & 0x00AA00AA00AA00AAull;  x = x ^ t ^ (t << 7);
  t = (x ^ (x >> 14)) & 0x0000CCCC0000CCCCull; x = x ^ t ^ (t << 14);
  t = (x ^ (x >> 28)) & 0x00000000F0F0F0F0ull; x = x ^ t ^ (t << 28);
  return x;
}

__device__ __forceinline__ uint32_t block_bytes(uint32_t F, int L) { return F == 0 ? 0u : (F + 1u) * uint32_t(L / 8); }

// ---------------------------------------------------------------- compress
template <int L>
__global__ void __launch_bounds__(kSThreads) small_sizes_kernel(CompressArgs a) {
  constexpr int kBlocks = kSTileElems / L;                 // L-blocks per tile
  static_assert(kBlocks % kSThreads == 0, "tile geometry");
  const float eb = resolve_eb(a);
  const bool eb_ok = eb_usable(eb);
  const float two_eb = __fadd_rn(eb, eb);
  const float recip = __fdiv_rn(1.0f, two_eb);
  const uint64_t t = blockIdx.x;
  uint32_t bytes = 0;
  bool bad = !eb_ok;
  if (eb_ok) {
    constexpr int kPer = kBlocks / kSThreads;
    float v[kPer][L];
#pragma unroll
    for (int j = 0; j < kPer; ++j) {                        // every load in flight before any math
      const uint64_t k = t * kBlocks + uint64_t(threadIdx.x + j * kSThreads);
      if (k < a.nb) block_load<L>(a.in, a.n, k, v[j]);
    }
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
      const uint64_t k = t * kBlocks + uint64_t(threadIdx.x + j * kSThreads);
      if (k >= a.nb) break;
      uint32_t mag[L], sign;
      const int F = block_encode<L>(v[j], eb, two_eb, recip, mag, sign, bad);
      a.out[kHdr + k] = uint8_t(F > kMaxF ? 0 : F);
      bytes += block_bytes(uint32_t(F), L);
    }
  }
  uint32_t total;
  cta_excl_scan(bytes, &total);
  if (__syncthreads_or(bad) && threadIdx.x == 0) atomicOr(&a.ws->status_accum, kBadRange);
  if (threadIdx.x == 0) a.status[t] = total;
}

// One CTA, in place: exclusive scan of the T tile sums.  Each thread owns a
// contiguous chunk (its loads are independent, so the whole array is one
// round of memory latency), chunk sums are scanned across the CTA, then
// written back as exclusive prefixes.  Returns the total (every thread).
__device__ __forceinline__ uint64_t tile_scan(uint64_t* st, uint64_t T, uint64_t* s_warp) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t per = (T + kScanThreads - 1) / kScanThreads;
  const uint64_t b = min(T, per * threadIdx.x), e = min(T, b + per);
  uint64_t v = 0;
  for (uint64_t i = b; i < e; ++i) v += st[i];
  uint64_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_warp[warp] = x;
  __syncthreads();
  uint64_t wb = 0, sum = 0;
  for (int w = 0; w < kScanThreads / 32; ++w) {
    if (w < warp) wb += s_warp[w];
    sum += s_warp[w];
  }
  uint64_t run = wb + x - v;
  for (uint64_t i = b; i < e; ++i) {
    const uint64_t c = st[i];
    st[i] = run;
    run += c;
  }
  __syncthreads();
  return sum;
}

// One CTA: exclusive scan of the tile byte sums in place, then the header.
template <int L>
__global__ void __launch_bounds__(kScanThreads) small_scan_kernel(CompressArgs a) {
  __shared__ uint64_t s_warp[kScanThreads / 32];
  __shared__ uint64_t s_carry;
  const uint32_t acc = *reinterpret_cast<volatile uint32_t*>(&a.ws->status_accum);
  const uint32_t status = (a.n > 0 && (acc & kBadRange)) ? CUSZP_ERANGE : CUSZP_OK;
  if (threadIdx.x == 0) s_carry = 0;
  __syncthreads();
  if (status == CUSZP_OK) {
    const uint64_t tot = tile_scan(a.status, a.num_tiles, s_warp);
    if (threadIdx.x == 0) s_carry = tot;
    __syncthreads();
  }
  if (threadIdx.x < 16 && a.nb + threadIdx.x < align16(a.nb))
    a.out[kHdr + a.nb + threadIdx.x] = 0;                  // F-area padding (R10)
  if (threadIdx.x == 0) {
    const float eb = resolve_eb(a);
    const uint64_t payload = status == CUSZP_OK ? s_carry : 0;
    const uint64_t p0 = kHdr + align16(a.nb);
    uint8_t* h = a.out;                                      // header (R10)
    *reinterpret_cast<uint32_t*>(h) = 0x505A5343u;           // "CSZP"
    h[4] = CUSZP_VERSION;
    h[5] = uint8_t(a.mode);
    h[6] = uint8_t(status);
    h[7] = uint8_t(L == 8 ? 3 : 4);                          // log2(L)
    *reinterpret_cast<uint64_t*>(h + 8) = a.n;
    *reinterpret_cast<float*>(h + 16) = a.mode == CUSZP_REL ? eb : a.eb_in;
    *reinterpret_cast<float*>(h + 20) = a.eb_in;
    *reinterpret_cast<uint64_t*>(h + 24) = payload;
    if (a.out_bytes) *a.out_bytes = (a.n == 0) ? uint64_t(kHdr) : p0 + payload;
    a.ws->last_status = status;
    a.ws->status_accum = 0;
    __threadfence();
  }
}

template <int L>
__global__ void __launch_bounds__(kSThreads) small_write_kernel(CompressArgs a) {
  constexpr int kBlocks = kSTileElems / L;
  constexpr int kPer = kBlocks / kSThreads;                 // blocks per thread (contiguous)
  constexpr int kPB = L / 8;                                // bytes per plane
  if (a.out[6] != CUSZP_OK) return;
  const float eb = resolve_eb(a);
  const float two_eb = __fadd_rn(eb, eb);
  const float recip = __fdiv_rn(1.0f, two_eb);
  const uint64_t t = blockIdx.x;
  const uint64_t k0 = t * kBlocks + uint64_t(threadIdx.x) * kPer;
  float v[kPer][L];                                         // input loads in flight during the scan
#pragma unroll
  for (int j = 0; j < kPer; ++j)
    if (k0 + j < a.nb) block_load<L>(a.in, a.n, k0 + j, v[j]);
  uint32_t bytes = 0;
#pragma unroll
  for (int j = 0; j < kPer; ++j)
    if (k0 + j < a.nb) bytes += block_bytes(a.out[kHdr + k0 + j], L);
  __shared__ __align__(16) uint8_t s_pay[kBlocks * kPB * (kMaxF + 1) + 16];   // the tile's payload
  uint8_t* dst = a.out + kHdr + align16(a.nb) + a.status[t];
  const uint32_t mis = uint32_t(reinterpret_cast<uintptr_t>(dst) & 3u);   // staged at dst's word phase
  uint32_t total;
  uint32_t off = mis + cta_excl_scan(bytes, &total);
  bool bad = false;
  for (int j = 0; j < kPer; ++j) {
    const uint64_t k = k0 + j;
    if (k >= a.nb) break;
    uint32_t mag[L], sign;
    const int F = block_encode<L>(v[j], eb, two_eb, recip, mag, sign, bad);
    if (F == 0) continue;                                   // zero block: F byte only (R6)
    uint8_t* o = s_pay + off;
#pragma unroll
    for (int b = 0; b < kPB; ++b) o[b] = uint8_t(sign >> (8 * b));   // sign map (R7, R9)
    for (int g = 0; 8 * g < F; ++g) {                       // block bit-shuffle, 8 planes at a time
#pragma unroll
      for (int b = 0; b < kPB; ++b) {                       // elements 8b .. 8b+7 -> byte b of each plane
        uint64_t x = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) x |= uint64_t((mag[8 * b + i] >> (8 * g)) & 0xffu) << (8 * i);
        x = transpose8(x);
        const int np = min(8, F - 8 * g);
        for (int q = 0; q < np; ++q) o[kPB * (1 + 8 * g + q) + b] = uint8_t(x >> (8 * q));
      }
    }
    off += block_bytes(uint32_t(F), L);
  }
  __syncthreads();
  // coalesced copy-out in words; the two edge words are shared with the
  // neighbouring tiles and go byte by byte
  uint8_t* dst_al = dst - mis;
  const uint32_t end = mis + total, nw = (end + 3) / 4;
  for (uint32_t w = threadIdx.x; w < nw; w += kSThreads) {
    if (4 * w >= mis && 4 * w + 4 <= end) {
      reinterpret_cast<uint32_t*>(dst_al)[w] = reinterpret_cast<const uint32_t*>(s_pay)[w];
    } else {
      for (uint32_t i = 4 * w; i < 4 * w + 4; ++i)
        if (i >= mis && i < end) dst_al[i] = s_pay[i];
    }
  }
}

// -------------------------------------------------------------- decompress
template <int L>
__device__ __forceinline__ uint32_t header_status(const DecompressArgs& a, float* eb_out, uint64_t* pbytes) {
  const uint64_t p0 = kHdr + align16(a.nb);
  if (a.in_bytes < uint64_t(kHdr)) return CUSZP_ECORRUPT;
  const uint8_t* h = a.in;
  const uint32_t magic = *reinterpret_cast<const uint32_t*>(h);
  const uint64_t hn = *reinterpret_cast<const uint64_t*>(h + 8);
  const float eb = *reinterpret_cast<const float*>(h + 16);
  *pbytes = *reinterpret_cast<const uint64_t*>(h + 24);
  *eb_out = eb;
  if (magic != 0x505A5343u || h[4] != CUSZP_VERSION || h[7] != uint8_t(L == 8 ? 3 : 4) || (h[5] & 0x10) != 0)
    return CUSZP_ECORRUPT;
  if (h[6] != CUSZP_OK) return h[6] == CUSZP_ERANGE ? CUSZP_ERANGE : CUSZP_ECORRUPT;
  if (hn != a.n) return CUSZP_EINVAL;
  if (a.n > 0) {
    if (!eb_usable(eb)) return CUSZP_ECORRUPT;
    if (a.in_bytes < p0 || a.in_bytes - p0 < *pbytes) return CUSZP_ECORRUPT;
  }
  return CUSZP_OK;
}

template <int L>
__global__ void __launch_bounds__(kSThreads) small_dsizes_kernel(DecompressArgs a) {
  constexpr int kBlocks = kSTileElems / L;
  float eb;
  uint64_t pbytes;
  if (header_status<L>(a, &eb, &pbytes) != CUSZP_OK) return;
  const uint64_t t = blockIdx.x;
  uint32_t bytes = 0;
  bool bad = false;
  for (int j = threadIdx.x; j < kBlocks; j += kSThreads) {
    const uint64_t k = t * kBlocks + uint64_t(j);
    if (k >= a.nb) break;
    const uint32_t F = a.in[kHdr + k];
    if (F > uint32_t(kMaxF)) bad = true;
    else bytes += block_bytes(F, L);
  }
  uint32_t total;
  cta_excl_scan(bytes, &total);
  if (__syncthreads_or(bad) && threadIdx.x == 0) atomicOr(&a.ws->status_accum, kBadCorrupt);
  if (threadIdx.x == 0) a.status[t] = total;
}

template <int L>
__global__ void __launch_bounds__(kScanThreads) small_dscan_kernel(DecompressArgs a) {
  __shared__ uint64_t s_warp[kScanThreads / 32];
  __shared__ uint64_t s_carry;
  float eb;
  uint64_t pbytes = 0;
  uint32_t status = header_status<L>(a, &eb, &pbytes);
  const uint32_t acc = *reinterpret_cast<volatile uint32_t*>(&a.ws->status_accum);
  if (status == CUSZP_OK && (acc & kBadCorrupt)) status = CUSZP_ECORRUPT;
  if (threadIdx.x == 0) s_carry = 0;
  __syncthreads();
  if (status == CUSZP_OK && a.n > 0) {
    const uint64_t tot = tile_scan(a.status, a.num_tiles, s_warp);
    if (threadIdx.x == 0) s_carry = tot;
    __syncthreads();
    if (s_carry != pbytes) status = CUSZP_ECORRUPT;       // Eq 3 total vs the header
  }
  if (threadIdx.x == 0) {
    a.ws->last_status = status;
    a.ws->status_accum = 0;
    __threadfence();
  }
}

template <int L>
__global__ void __launch_bounds__(kSThreads) small_decode_kernel(DecompressArgs a) {
  constexpr int kBlocks = kSTileElems / L;
  constexpr int kPer = kBlocks / kSThreads;
  constexpr int kPB = L / 8;
  if (*reinterpret_cast<volatile uint32_t*>(&a.ws->last_status) != CUSZP_OK) return;
  const float eb = *reinterpret_cast<const float*>(a.in + 16);
  const float two_eb = __fadd_rn(eb, eb);
  const uint64_t t = blockIdx.x;
  const uint64_t k0 = t * kBlocks + uint64_t(threadIdx.x) * kPer;
  uint32_t bytes = 0;
#pragma unroll
  for (int j = 0; j < kPer; ++j)
    if (k0 + j < a.nb) bytes += block_bytes(a.in[kHdr + k0 + j], L);
  __shared__ __align__(16) uint8_t s_pay[kBlocks * kPB * (kMaxF + 1) + 16];
  const uint8_t* src = a.in + kHdr + align16(a.nb) + a.status[t];
  const uint32_t mis = uint32_t(reinterpret_cast<uintptr_t>(src) & 3u);
  uint32_t total;
  uint32_t off = mis + cta_excl_scan(bytes, &total);
  // coalesced copy-in of whole aligned words; the leading edge word's extra
  // bytes precede this tile's payload inside the stream, the trailing edge
  // word is copied byte by byte so no read passes the tile's last byte (the
  // stream may end there: in_bytes bounds every read, cuszp.h)
  const uint32_t end = mis + total;
  const uint32_t nfull = end / 4;
  const uint32_t* src_al = reinterpret_cast<const uint32_t*>(src - mis);
  for (uint32_t w = threadIdx.x; w < nfull; w += kSThreads) reinterpret_cast<uint32_t*>(s_pay)[w] = src_al[w];
  if (threadIdx.x < (end & 3u)) s_pay[4 * nfull + threadIdx.x] = (src - mis)[4 * nfull + threadIdx.x];
  __syncthreads();
  for (int j = 0; j < kPer; ++j) {
    const uint64_t k = k0 + j;
    if (k >= a.nb) break;
    const uint32_t F = a.in[kHdr + k];
    const uint8_t* p = s_pay + off;
    uint32_t sign = 0;
    uint32_t mag[L];
#pragma unroll
    for (int i = 0; i < L; ++i) mag[i] = 0;
    if (F > 0) {
#pragma unroll
      for (int b = 0; b < kPB; ++b) sign |= uint32_t(p[b]) << (8 * b);
      for (int g = 0; 8 * g < int(F); ++g) {                // inverse bit-shuffle, 8 planes at a time
        const int np = min(8, int(F) - 8 * g);
#pragma unroll
        for (int b = 0; b < kPB; ++b) {
          uint64_t x = 0;
          for (int q = 0; q < np; ++q) x |= uint64_t(p[kPB * (1 + 8 * g + q) + b]) << (8 * q);
          x = transpose8(x);
#pragma unroll
          for (int i = 0; i < 8; ++i) mag[8 * b + i] |= uint32_t((x >> (8 * i)) & 0xffu) << (8 * g);
        }
      }
    }
    int32_t r = 0;                                         // reverse Lorenzo
    float y[L];
#pragma unroll
    for (int i = 0; i < L; ++i) {
      r += ((sign >> i) & 1u) ? -int32_t(mag[i]) : int32_t(mag[i]);
      y[i] = __fmul_rn(float(r), two_eb);                  // d' = r * 2eb
    }
    if ((k + 1) * L <= a.n) {                              // whole block: 16-byte stores
      float4* o = reinterpret_cast<float4*>(a.out + k * L);
#pragma unroll
      for (int q = 0; q < L / 4; ++q) o[q] = make_float4(y[4 * q], y[4 * q + 1], y[4 * q + 2], y[4 * q + 3]);
    } else {
#pragma unroll
      for (int i = 0; i < L; ++i)
        if (k * L + uint64_t(i) < a.n) a.out[k * L + i] = y[i];
    }
    off += block_bytes(F, L);
  }
}

template <int L>
cudaError_t compress_small(const CompressArgs& a, cudaStream_t s) {
  if (a.num_tiles > 0) small_sizes_kernel<L><<<a.num_tiles, kSThreads, 0, s>>>(a);
  small_scan_kernel<L><<<1, kScanThreads, 0, s>>>(a);
  if (a.num_tiles > 0) small_write_kernel<L><<<a.num_tiles, kSThreads, 0, s>>>(a);
  return cudaGetLastError();
}

template <int L>
cudaError_t decompress_small(const DecompressArgs& a, cudaStream_t s) {
  if (a.num_tiles > 0) small_dsizes_kernel<L><<<a.num_tiles, kSThreads, 0, s>>>(a);
  small_dscan_kernel<L><<<1, kScanThreads, 0, s>>>(a);
  if (a.num_tiles > 0) small_decode_kernel<L><<<a.num_tiles, kSThreads, 0, s>>>(a);
  return cudaGetLastError();
}

}  // namespace

cudaError_t compress_small_launch(int L, const CompressArgs& a, cudaStream_t s) {
  return L == 8 ? compress_small<8>(a, s) : compress_small<16>(a, s);
}

cudaError_t decompress_small_launch(int L, const DecompressArgs& a, cudaStream_t s) {
  return L == 8 ? decompress_small<8>(a, s) : decompress_small<16>(a, s);
}

}  // namespace cuszp

#endif  // CUSZP_SMALL_L_3PASS
