// decompress.cu -- the fused cuSZp decompression kernel for sm_100a
// (paper sec 3.2 / Fig 3).
//
// Per 2048-element tile taken by ticket:
//   a9  fixed lengths F -> CmpL (Eq 2) -> the same hierarchical scan +
//       decoupled look-back as compression
//   a10 inverse bit-shuffle: lane k holds word k of the block (sign map,
//       then planes); lane j gathers bit j of every plane, applies the sign
//   a11 inverse Lorenzo: 32-lane inclusive scan (5 x shfl_up)
//   a12 dequantise d' = (float)r * 2eb (R13), coalesced store
// Every read is bounded by in_bytes (corrupt input -> async ECORRUPT).
#include "internal.cuh"

namespace cuszp {

__global__ void __launch_bounds__(kThreads) decompress_kernel(DecompressArgs a) {
  __shared__ uint32_t s_tile;
  __shared__ uint32_t s_warp_words[kWarps];
  __shared__ uint64_t s_warp_base[kWarps];

  const int lane = threadIdx.x & 31;
  const int warp = threadIdx.x >> 5;
  const uint32_t epoch = running_epoch(a.ws);

  // ---- header (R10), validated identically by every CTA
  uint32_t err = CUSZP_OK;
  float eb = 0.0f;
  uint64_t payload_words = 0;
  const uint64_t p0 = kHdr + align16(a.nb);
  if (a.in_bytes < uint64_t(kHdr)) {
    err = CUSZP_ECORRUPT;
  } else {
    const uint8_t* h = a.in;
    const uint32_t magic = *reinterpret_cast<const uint32_t*>(h);
    const uint64_t hn = *reinterpret_cast<const uint64_t*>(h + 8);
    eb = *reinterpret_cast<const float*>(h + 16);
    const uint64_t pbytes = *reinterpret_cast<const uint64_t*>(h + 24);
    if (magic != 0x505A5343u || h[4] != CUSZP_VERSION || h[7] != 5) err = CUSZP_ECORRUPT;
    else if (h[6] != CUSZP_OK) err = (h[6] == CUSZP_ERANGE) ? CUSZP_ERANGE : CUSZP_ECORRUPT;
    else if (hn != a.n) err = CUSZP_EINVAL;
    else if (a.n > 0) {
      const float two = __fadd_rn(eb, eb);
      if (!(eb >= kFltMin) || !isfinite(two)) err = CUSZP_ECORRUPT;
      else if ((pbytes & 3u) || a.in_bytes < p0 || a.in_bytes - p0 < pbytes) err = CUSZP_ECORRUPT;
      payload_words = pbytes / 4;
    }
  }
  const float two_eb = __fadd_rn(eb, eb);
  const uint32_t* payload = reinterpret_cast<const uint32_t*>(a.in + p0);
  uint32_t bad = 0;

  if (err == CUSZP_OK && a.n > 0) {
    while (true) {
      if (threadIdx.x == 0) s_tile = atomicAdd(&a.ws->ticket, 1u);
      __syncthreads();
      const uint32_t t = s_tile;
      if (t >= a.num_tiles) break;

      const uint64_t blk0 = uint64_t(t) * kTileBlocks + uint64_t(warp) * kBPW;
      // -- fixed lengths of the warp's 8 blocks (one 8-byte read, R10 padding keeps it in bounds)
      uint64_t fw = 0;
      if (blk0 < a.nb) fw = *reinterpret_cast<const uint64_t*>(a.in + kHdr + blk0);
      uint32_t F[kBPW], pre[kBPW];
      uint32_t wsum = 0;
#pragma unroll
      for (int b = 0; b < kBPW; ++b) {
        uint32_t f = uint32_t(fw >> (8 * b)) & 0xffu;
        if (blk0 + b >= a.nb) f = 0;
        if (f > uint32_t(kMaxF)) { bad |= kBadCorrupt; f = 0; }
        F[b] = f;
        pre[b] = wsum;
        wsum += f ? f + 1u : 0u;                        // Eq 2 in 4-byte words
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
        const uint64_t excl = tile_lookback(a.status, t, agg, epoch);
        if (lane < kWarps) s_warp_base[lane] = excl + incl - v;
      }
      __syncthreads();
      const uint64_t base = s_warp_base[warp];

      // -- gather the payload words: lane k <- word k of block b
      uint32_t word[kBPW];
#pragma unroll
      for (int b = 0; b < kBPW; ++b) {
        word[b] = 0;
        const uint64_t wi = base + pre[b] + lane;
        if (F[b] != 0 && uint32_t(lane) <= F[b]) {
          if (wi < payload_words) word[b] = __ldg(payload + wi);
          else bad |= kBadCorrupt;
        }
      }
#pragma unroll
      for (int b = 0; b < kBPW; ++b) {
        const uint32_t f = F[b];
        // a10: |l_j| = sum_k bit_j(plane_k) << k, sign from the sign map
        const uint32_t sign = __shfl_sync(kFull, word[b], 0);
        uint32_t mag = 0;
        for (int k = int(f); k >= 1; --k) {
          const uint32_t plane = __shfl_sync(kFull, word[b], k);
          mag = (mag << 1) | ((plane >> lane) & 1u);
        }
        int l = int(mag);
        if ((sign >> lane) & 1u) l = -l;
        // a11: r_j = sum_{i<=j} l_i inside the block
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(kFull, l, o);
          if (lane >= o) l += y;
        }
        // a12: d' = r * 2eb
        const float d = __fmul_rn(__int2float_rn(l), two_eb);
        const uint64_t idx = (blk0 + b) * kL + lane;
        if (idx < a.n) a.out[idx] = d;
      }
    }
  }

  if (cta_finish(a.ws, bad)) {
    uint32_t final_status = err;
    if (threadIdx.x == 0 && final_status == CUSZP_OK) {
      const uint32_t acc = *reinterpret_cast<volatile uint32_t*>(&a.ws->status_accum);
      if (acc & kBadCorrupt) final_status = CUSZP_ECORRUPT;
      if (final_status == CUSZP_OK && a.num_tiles > 0 && a.n > 0) {
        const uint64_t total = ld_relaxed_u64(a.status + a.num_tiles - 1) & kValueMask;
        if (total != payload_words) final_status = CUSZP_ECORRUPT;
      }
    }
    finish_call(a.ws, a.status, a.status_cap, epoch, final_status);
  }
}

}  // namespace cuszp
