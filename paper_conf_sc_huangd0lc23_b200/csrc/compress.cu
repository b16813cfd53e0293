// compress.cu -- the fused cuSZp compression kernel for sm_100a
// (paper sec 3.1 / Fig 2 and sec 4).
//
// One launch does, per 2048-element tile taken by ticket:
//   a2 pre-quantisation   r = round(d / 2eb)              (R2)
//   a3 block Lorenzo      l_j = r_j - r_{j-1}, r_{-1}=0
//   a4 sign map           ballot(l < 0)                    (R7)
//   a5 fixed length       F = 32 - clz(redux.max |l|)
//   a6 CmpL               4 (F + 1) bytes, 0 if F = 0      (Eq 2, R6)
//   a7 global sync        warp / CTA prefix + decoupled look-back (Eq 3,
//                         hierarchy of Fig 9)
//   a8 bit-shuffle        plane k = ballot(bit k of |l|), stored with the
//                         sign map at the scanned offset   (R9)
// Layout in the output stream: DESIGN.md sec 4.
#include "internal.cuh"

namespace cuszp {

namespace {

// Quantise one element with the R2 op sequence (explicit RN intrinsics:
// never contracted, identical to the oracle's separately rounded ops).
__device__ __forceinline__ int quantize(float x, float eb, float two_eb, float recip, bool& ok) {
  const float v = __fmul_rn(x, recip);
  ok = fabsf(v) < kGuard;                               // NaN / Inf / overflow -> false (R5)
  const float t = __fadd_rn(v, kRoundMagic);           // = 1.5*2^23 + rint(v), |v| < 2^22
  const float r0 = __fsub_rn(t, kRoundMagic);          // rint(v), exact
  const float res = __fmaf_rn(-r0, two_eb, x);         // d - r0*2eb, exact (R2)
  int r = int(__float_as_uint(t) - kRoundMagicBits);   // rint(v) as an integer
  r += int(res > eb) - int(res < -eb);
  return r;
}

}  // namespace

__global__ void __launch_bounds__(kThreads) compress_kernel(CompressArgs a) {
  __shared__ uint32_t s_tile;
  __shared__ uint32_t s_warp_words[kWarps];
  __shared__ uint64_t s_warp_base[kWarps];

  const int lane = threadIdx.x & 31;
  const int warp = threadIdx.x >> 5;
  const uint32_t epoch = running_epoch(a.ws);

  // ---- resolve eb_abs (Eq 1): ABS -> delta; REL -> lambda * (max - min) over the pairs
  float eb = a.eb_in;
  if (a.mode == CUSZP_REL) {
    float mn = a.minmax[0], mx = a.minmax[1];
    bool nan = isnan(mn) || isnan(mx);
    for (int p = 1; p < a.n_pairs; ++p) {
      const float lo = a.minmax[2 * p], hi = a.minmax[2 * p + 1];
      nan |= isnan(lo) || isnan(hi);
      if (lo < mn) mn = lo;
      if (hi > mx) mx = hi;
    }
    eb = __fmul_rn(a.eb_in, __fsub_rn(mx, mn));         // R3
    if (nan) eb = __int_as_float(0x7fc00000);
  }
  const float two_eb = __fadd_rn(eb, eb);
  const bool eb_ok = (eb >= kFltMin) && isfinite(two_eb) && a.n > 0;   // R5
  const float recip = __fdiv_rn(1.0f, two_eb);

  uint32_t bad = (a.n > 0 && !eb_ok) ? kBadRange : 0u;
  const uint64_t p0 = kHdr + align16(a.nb);
  uint32_t* payload = reinterpret_cast<uint32_t*>(a.out + p0);

  if (eb_ok) {
    while (true) {
      if (threadIdx.x == 0) s_tile = atomicAdd(&a.ws->ticket, 1u);
      __syncthreads();
      const uint32_t t = s_tile;
      if (t >= a.num_tiles) break;

      const uint64_t blk0 = uint64_t(t) * kTileBlocks + uint64_t(warp) * kBPW;

      // -- load: lane j <- element j of each of the warp's 8 blocks (coalesced 128 B rows)
      float x[kBPW];
#pragma unroll
      for (int b = 0; b < kBPW; ++b) {
        const uint64_t idx = (blk0 + b) * kL + lane;
        x[b] = idx < a.n ? ld_stream_f32(a.in + idx) : 0.0f;    // virtual zero pad (R8)
      }

      // -- per block: quantise, predict, encode (all in registers)
      uint32_t word[kBPW];   // lane 0: sign map, lane k+1: plane k
      uint32_t F[kBPW];      // warp-uniform
#pragma unroll
      for (int b = 0; b < kBPW; ++b) {
        bool ok;
        const int r = quantize(x[b], eb, two_eb, recip, ok);
        if (!ok && (blk0 + b) * kL + lane < a.n) bad |= kBadRange;
        const int prev = __shfl_up_sync(kFull, r, 1);
        const int l = (lane == 0) ? r : r - prev;
        const uint32_t sign = __ballot_sync(kFull, l < 0);
        const uint32_t mag = uint32_t(l < 0 ? -l : l);
        const uint32_t m = __reduce_max_sync(kFull, mag);
        const uint32_t f = 32u - __clz(m);
        uint32_t w = sign;
        for (uint32_t k = 0; k < f; ++k) {
          const uint32_t plane = __ballot_sync(kFull, (mag >> k) & 1u);
          if (lane == int(k) + 1) w = plane;
        }
        word[b] = w;
        F[b] = f;
      }

      // -- hierarchical scan (Fig 9): thread/warp level is a serial sum of the warp's 8 blocks
      uint32_t pre[kBPW];
      uint32_t wsum = 0;
#pragma unroll
      for (int b = 0; b < kBPW; ++b) {
        pre[b] = wsum;
        wsum += F[b] ? F[b] + 1u : 0u;
      }
      if (lane == 0) s_warp_words[warp] = wsum;
      __syncthreads();
      if (warp == 0) {
        const uint32_t v = lane < kWarps ? s_warp_words[lane] : 0u;
        uint32_t incl = v;
#pragma unroll
        for (int o = 1; o < kWarps; o <<= 1) {
          const uint32_t y = __shfl_up_sync(kFull, incl, o);
          if (lane >= o) incl += y;
        }
        const uint32_t agg = __shfl_sync(kFull, incl, kWarps - 1);
        const uint64_t excl = tile_lookback(a.status, t, agg, epoch);   // global level
        if (lane < kWarps) s_warp_base[lane] = excl + incl - v;
      }
      __syncthreads();
      const uint64_t base = s_warp_base[warp];

      // -- fixed-length bytes (Fig 12 part 1): 8 blocks -> two u32 stores
      if (lane < 2 && blk0 + 4 * lane < align16(a.nb)) {
        const uint32_t lo = F[0] | (F[1] << 8) | (F[2] << 16) | (F[3] << 24);
        const uint32_t hi = F[4] | (F[5] << 8) | (F[6] << 16) | (F[7] << 24);
        *reinterpret_cast<uint32_t*>(a.out + kHdr + blk0 + 4 * lane) = lane ? hi : lo;
      }
      // -- shuffled bytes at the synchronised offsets (Fig 12 part 2)
#pragma unroll
      for (int b = 0; b < kBPW; ++b) {
        if (F[b] != 0 && uint32_t(lane) <= F[b]) payload[base + pre[b] + lane] = word[b];
      }
    }
  }

  if (cta_finish(a.ws, bad)) {
    uint32_t final_status = CUSZP_OK;
    uint64_t total_words = 0;
    if (threadIdx.x == 0) {
      const uint32_t acc = *reinterpret_cast<volatile uint32_t*>(&a.ws->status_accum);
      if (acc & kBadRange) final_status = CUSZP_ERANGE;
      if (final_status == CUSZP_OK && a.num_tiles > 0)
        total_words = ld_relaxed_u64(a.status + a.num_tiles - 1) & kValueMask;
      const uint64_t payload_bytes = final_status == CUSZP_OK ? total_words * 4 : 0;
      // header (R10)
      uint8_t* h = a.out;
      *reinterpret_cast<uint32_t*>(h) = 0x505A5343u;   // "CSZP"
      h[4] = CUSZP_VERSION;
      h[5] = uint8_t(a.mode);
      h[6] = uint8_t(final_status);
      h[7] = 5;
      *reinterpret_cast<uint64_t*>(h + 8) = a.n;
      *reinterpret_cast<float*>(h + 16) = a.n > 0 ? eb : (a.mode == CUSZP_REL ? 0.0f : a.eb_in);
      *reinterpret_cast<float*>(h + 20) = a.eb_in;
      *reinterpret_cast<uint64_t*>(h + 24) = payload_bytes;
      if (a.out_bytes)
        *a.out_bytes = (a.n == 0) ? uint64_t(kHdr) : p0 + payload_bytes;
    }
    finish_call(a.ws, a.status, a.status_cap, epoch, final_status);
  }
}

}  // namespace cuszp
