// decompress.cu -- the fused cuSZp decompression kernel for sm_100a
// (paper sec 3.2 / Fig 3).
//
// Persistent, warp-specialised CTA:
//   warps 0..3  producers, one per ring stage (4 tiles in flight per CTA):
//               take a tile ticket, read the tile's 128 fixed-length bytes,
//               turn them into block word counts (Eq 2) and tile-local
//               offsets (warp scan), publish the tile aggregate at once,
//               resolve the tile's global offset with the decoupled look-back
//               (a9, Eq 3) and stream the tile's payload HBM -> shared memory
//               with one 1D TMA bulk copy;
//   warps 4..11 compute (stages consumed round-robin): 16 blocks each, two blocks per warp bit transpose
//               (lane k <- word k of block A, lane 16+k <- word k of block B;
//               afterwards lane j holds 2|l_j| + sign_j of both):
//     a10 inverse bit-shuffle + sign,
//     a11 inverse Lorenzo: four blocks are re-laid out through shared memory
//         (4 consecutive elements per lane, 8 lanes per block): 3 local adds
//         + a 3-step segmented shuffle scan,
//     a12 dequantise d' = (float) r * 2eb (R13), 128-bit stores.
// Every read is bounded by in_bytes (corrupt input -> async ECORRUPT).
#include "internal.cuh"

namespace cuszp {

namespace {

#ifndef CUSZP_D_MINBLOCKS
#define CUSZP_D_MINBLOCKS 3
#endif
#ifndef CUSZP_D_STAGES
#define CUSZP_D_STAGES 4
#endif
constexpr int kDStages = CUSZP_D_STAGES;
constexpr int kDataWords = kTileBlocks * kMaxBlockWords + 8;   // 3208 words: worst tile + alignment slack
constexpr int kDThreads = (kDStages + kComputeWarps) * 32;

struct DecompressSmem {
  uint32_t data[kDStages][kDataWords];         // 51.3 KB
  uint16_t boff[kDStages][kTileBlocks];        // tile-local word offset of each block
  uint8_t bwords[kDStages][kTileBlocks];       // words per block: F + 1, or 0
  uint32_t tile[kDStages];
  uint32_t delta[kDStages];                    // first payload word of the tile inside data[]
  alignas(16) int scratch[kComputeWarps][8 * 32];   // per-warp 8-block re-layout for the scan
  uint64_t full[kDStages], empty[kDStages];
};

}  // namespace

__global__ void __launch_bounds__(kDThreads, CUSZP_D_MINBLOCKS) decompress_kernel(DecompressArgs a) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  DecompressSmem& sm = *reinterpret_cast<DecompressSmem*>(smem_raw);
  const int lane = threadIdx.x & 31;
  const int warp = threadIdx.x >> 5;
  const uint32_t epoch = running_epoch(a.ws);

  // ---- header (R10), validated identically by every thread
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
  uint32_t bad = 0;

  if (threadIdx.x == 0) {
    for (int s = 0; s < kDStages; ++s) { mbar_init(&sm.full[s], 1); mbar_init(&sm.empty[s], kComputeWarps); }
    fence_mbar_init();
  }
  __syncthreads();

  if (err == CUSZP_OK && a.n > 0) {
    if (warp < kDStages) {
      // ------------------------------------------- producers (one per stage)
      const int s = warp;
      for (uint32_t j = 0;; ++j) {
        mbar_wait(&sm.empty[s], (j & 1u) ^ 1u);
        uint32_t t = 0;
        if (lane == 0) t = atomicAdd(&a.ws->ticket, 1u);
        t = __shfl_sync(kFull, t, 0);
        if (lane == 0 && t < a.num_tiles) trace_put(a.trace, t, 0, global_ns());
        if (t >= a.num_tiles) {
          if (lane == 0) {
            sm.tile[s] = kSentinel;
            mbar_arrive(&sm.full[s]);
          }
          break;
        }
        // a9: fixed lengths -> words per block (Eq 2) -> tile-local offsets
        const uint64_t blk = uint64_t(t) * kTileBlocks + 4u * lane;   // this lane's 4 blocks
        uint32_t fq = 0;
        if (blk < a.nb) fq = *reinterpret_cast<const uint32_t*>(a.in + kHdr + blk);
        uint32_t wq[4], lsum = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          uint32_t f = (fq >> (8 * k)) & 0xffu;
          if (blk + k >= a.nb) f = 0;
          if (f > uint32_t(kMaxF)) { bad |= kBadCorrupt; f = 0; }
          wq[k] = f ? f + 1 : 0;
          lsum += wq[k];
        }
        uint32_t incl = lsum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(kFull, incl, o);
          if (lane >= o) incl += y;
        }
        const uint32_t agg = __shfl_sync(kFull, incl, 31);
        uint32_t o0 = incl - lsum;
        const uint32_t o1 = o0 + wq[0], o2 = o1 + wq[1], o3 = o2 + wq[2];
        *reinterpret_cast<uint2*>(&sm.boff[s][4 * lane]) = make_uint2(o0 | (o1 << 16), o2 | (o3 << 16));
        *reinterpret_cast<uint32_t*>(&sm.bwords[s][4 * lane]) = wq[0] | (wq[1] << 8) | (wq[2] << 16) | (wq[3] << 24);
        // a9: global synchronisation (decoupled look-back)
        if (lane == 0) publish_aggregate(a.status, t, agg, epoch);
        uint32_t nw = 0, ns = 0;
        const uint64_t t_lb = a.trace ? global_ns() : 0;
        const uint64_t excl = resolve_prefix(a.status, t, agg, epoch, &nw, &ns);
        if (lane == 0 && a.trace) {
          // decompress trace: 0 ticket, 1 F loaded + A published, 2 prefix, 3 TMA issued,
          // 4 first compute pickup, 5 last compute done, 6 windows<<32|spins, 7 smid<<32|cta
          trace_put(a.trace, t, 1, t_lb);
          trace_put(a.trace, t, 2, global_ns());
          trace_put(a.trace, t, 6, (uint64_t(nw) << 32) | ns);
          uint32_t smid;
          asm("mov.u32 %0, %smid;" : "=r"(smid));
          trace_put(a.trace, t, 7, (uint64_t(smid) << 32) | blockIdx.x);
        }
        uint32_t tma_bytes = 0, delta = 0;
        if (excl + agg > payload_words) {
          bad |= kBadCorrupt;   // offsets beyond the stream: decode zeros, never read out of bounds
          *reinterpret_cast<uint32_t*>(&sm.bwords[s][4 * lane]) = 0u;
        } else if (agg > 0) {
          const uint64_t start = p0 + 4 * excl, end = start + 4ull * agg;
          const uint64_t a0 = start & ~uint64_t(15);
          uint64_t a1 = (end + 15) & ~uint64_t(15);
          if (a1 > a.in_bytes) a1 = a.in_bytes & ~uint64_t(15);
          tma_bytes = uint32_t(a1 - a0);
          delta = uint32_t(start - a0) / 4;
          // words past the last full 16 bytes inside in_bytes (<= 3)
          const uint64_t tail_words = end > a1 ? (end - a1) / 4 : 0;
          if (uint64_t(lane) < tail_words)
            sm.data[s][(a1 - a0) / 4 + lane] = *reinterpret_cast<const uint32_t*>(a.in + a1 + 4 * lane);
        }
        __syncwarp();
        if (lane == 0) {
          sm.tile[s] = t;
          sm.delta[s] = delta;
          mbar_arrive_expect_tx(&sm.full[s], tma_bytes);
          if (tma_bytes) tma_load_1d(sm.data[s], a.in + ((p0 + 4 * excl) & ~uint64_t(15)), tma_bytes, &sm.full[s]);
          trace_put(a.trace, t, 3, global_ns());
        }
      }
    } else {
      // ------------------------------------------------------------ compute
      const int w = warp - kDStages;
      const Xpose xpose(lane);
      const bool hi = lane >= 16;
      const uint32_t k16 = lane & 15;
      // Stages are consumed round-robin; each producer ends its stage with a
      // sentinel, so keep going until every stage has delivered one.
      // Each warp takes whichever stage is ready first (no head-of-line
      // blocking behind a stage whose look-back is still waiting).
      uint32_t phase = 0;   // bit s: parity of stage s's next phase
      uint32_t done = 0;
      int s = 0;
      for (;;) {
        // probe every pending stage once; if none is ready, sleep (in hardware)
        // on the next pending one until it completes
        int probes = 0;
        while (true) {
          if (!(done & (1u << s))) {
            if (probes < kDStages ? mbar_test(&sm.full[s], (phase >> s) & 1u)
                                  : mbar_try(&sm.full[s], (phase >> s) & 1u))
              break;
          }
          if (++probes < kDStages || (done & (1u << s))) s = (s + 1) % kDStages;
        }
        phase ^= 1u << s;
        const uint32_t t = sm.tile[s];
        if (t != kSentinel && lane == 0 && a.trace)
          atomicMin(reinterpret_cast<unsigned long long*>(a.trace + 8ull * t + 4), (unsigned long long)global_ns());
        if (t == kSentinel) {
          done |= 1u << s;
          if (done == (1u << kDStages) - 1) break;
          s = (s + 1) % kDStages;
          continue;
        }
        const bool last = (t == a.num_tiles - 1);
        const uint32_t* data = sm.data[s] + sm.delta[s];
        const uint64_t g0 = uint64_t(t) * kTileElems + uint64_t(w) * kBPW * 32;
        int* scratch = sm.scratch[w];
        // 16 blocks = 2 rounds of 8 (4 pairs each, independent transposes in flight)
#pragma unroll 1
        for (int g = 0; g < kBPW / 8; ++g) {
#pragma unroll
          for (int h = 0; h < 4; ++h) {
            const int lb = w * kBPW + 8 * g + 2 * h;
            const uint32_t offs = *reinterpret_cast<const uint32_t*>(&sm.boff[s][lb]);
            const uint32_t wds = *reinterpret_cast<const uint16_t*>(&sm.bwords[s][lb]);
            const uint32_t oa = offs & 0xffffu, ob = offs >> 16;
            const uint32_t wa = wds & 0xffu, wb = wds >> 8;
            uint32_t va, vb;
            if (wa <= 16 && wb <= 16) {
              // a10: lane k (< 16) <- word k of A, lane 16+k <- word k of B; one transpose
              const uint32_t idx = oa + (hi ? wa : 0u) + k16;
              const uint32_t x = (k16 < (hi ? wb : wa)) ? data[idx] : 0u;
              const uint32_t tw = xpose(x);
              va = tw & 0xffffu;
              vb = tw >> 16;
            } else {
              va = xpose(uint32_t(lane) < wa ? data[oa + lane] : 0u);
              vb = xpose(uint32_t(lane) < wb ? data[ob + lane] : 0u);
            }
            // sign: v = 2|l| + s  ->  l = s ? -|l| : |l|
            const int ma = int(va >> 1), mb = int(vb >> 1);
            scratch[(2 * h) * 32 + lane] = (va & 1u) ? -ma : ma;
            scratch[(2 * h + 1) * 32 + lane] = (vb & 1u) ? -mb : mb;
          }
          __syncwarp();
          // a11: 8 blocks, 4 consecutive elements per lane, 8 lanes per block, 2 passes
#pragma unroll
          for (int q = 0; q < 2; ++q) {
            int4 e = *reinterpret_cast<const int4*>(&scratch[(4 * q + (lane >> 3)) * 32 + 4 * (lane & 7)]);
            e.y += e.x;
            e.z += e.y;
            e.w += e.z;
            int incl = e.w;
            incl = scan_step_up(incl, 1, 24 << 8);
            incl = scan_step_up(incl, 2, 24 << 8);
            incl = scan_step_up(incl, 4, 24 << 8);
            const int carry = incl - e.w;
            e.x += carry; e.y += carry; e.z += carry; e.w += carry;
            // a12: d' = r * 2eb
            float4 d;
            d.x = __fmul_rn(__int2float_rn(e.x), two_eb);
            d.y = __fmul_rn(__int2float_rn(e.y), two_eb);
            d.z = __fmul_rn(__int2float_rn(e.z), two_eb);
            d.w = __fmul_rn(__int2float_rn(e.w), two_eb);
            const uint64_t i0 = g0 + uint64_t(8 * g + 4 * q + (lane >> 3)) * 32 + 4 * (lane & 7);
            if (!last || i0 + 4 <= a.n) {
              *reinterpret_cast<float4*>(a.out + i0) = d;
            } else {
              if (i0 < a.n) a.out[i0] = d.x;
              if (i0 + 1 < a.n) a.out[i0 + 1] = d.y;
              if (i0 + 2 < a.n) a.out[i0 + 2] = d.z;
            }
          }
          __syncwarp();
        }
        __syncwarp();
        if (lane == 0) {
          if (a.trace) atomicMax(reinterpret_cast<unsigned long long*>(a.trace + 8ull * t + 5), (unsigned long long)global_ns());
          mbar_arrive(&sm.empty[s]);
        }
        s = (s + 1) % kDStages;
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

size_t decompress_smem_bytes() { return sizeof(DecompressSmem); }
int decompress_threads() { return kDThreads; }

}  // namespace cuszp
