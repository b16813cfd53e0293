// decompress.cu -- the fused cuSZp decompression kernel for sm_100a
// (paper sec 3.2 / Fig 3).
//
// Persistent, warp-specialised CTA:
//   warp 0      scanner: takes a CHUNK ticket (4 tiles = 512 blocks), reads the
//               chunk's 512 fixed-length bytes (one 16-byte load per lane),
//               turns them into block word counts (Eq 2), per-group offsets
//               and packing modes, publishes the chunk aggregate and resolves
//               the chunk's global offset with the decoupled look-back (a9,
//               Eq 3) -- one look-back per 4 tiles, overlapped with decoding
//               through a double-buffered chunk descriptor;
//   warp 1      loader: streams every tile's payload HBM -> shared memory
//               with one 1D TMA bulk copy into a kDStages-deep ring;
//   warps 2..9  compute, 16 blocks each in groups of 4 -- four, two or one
//               blocks per warp bit transpose (8, 16 or 32 lanes per block):
//     a10 inverse bit-shuffle: lane k of a block's lane range <- word k
//         (sign map, then planes); after the transpose lane j holds
//         v_j = 2|l_j| + sign_j of each packed block; rows go to shared memory,
//     a11 inverse Lorenzo: 4 consecutive elements per lane, 8 lanes per block,
//         3 local adds + a 3-step segmented shuffle scan,
//     a12 dequantise d' = (float) r * 2eb (R13), 128-bit stores.
// L = 8 / 16 (SL): look-back units are bytes; the scanner sums the block
// bytes of whole warp slices, the loader also stages the tile's F bytes, and
// each compute lane decodes one block in registers.
// Every read is bounded by in_bytes (corrupt input -> async ECORRUPT).
#include <type_traits>

#include "internal.cuh"

namespace cuszp {

namespace {

#ifndef CUSZP_D_MINBLOCKS
#define CUSZP_D_MINBLOCKS 4   // 4 CTAs x 10 warps per SM: the decode is latency-bound (48 registers, no spills)
#endif
#ifndef CUSZP_D_STAGES
#define CUSZP_D_STAGES 2
#endif
constexpr int kDStages = CUSZP_D_STAGES;
#ifndef CUSZP_D_UNROLL
#define CUSZP_D_UNROLL 4
#endif
constexpr int kDUnroll = CUSZP_D_UNROLL;                        // decode groups interleaved per iteration
#ifndef CUSZP_D_CHUNK_TILES
#define CUSZP_D_CHUNK_TILES 8
#endif
// tiles per look-back unit: the scanner's latency per chunk (F loads + one
// look-back, ~2 + ~7 us under load) must stay below the CTA's decode time of
// the chunk (~1.8 us per tile), else the loader starves
constexpr int kChunkTiles = CUSZP_D_CHUNK_TILES;
static_assert(kChunkTiles == 4 || kChunkTiles == 8, "chunk of 4 or 8 tiles");
constexpr int kGroups = kTileBlocks / 4;                        // 32 decode groups per tile
constexpr int kDataWords = kTileBlocks * kMaxBlockWords + 8;   // 3208 words: worst tile + alignment slack
constexpr int kDFirstCompute = 2;
constexpr int kDThreads = (kDFirstCompute + kComputeWarps) * 32;

struct ChunkDesc {
  uint64_t tile_start[kChunkTiles];   // global payload word offset of each tile
  uint32_t tile_words[kChunkTiles];
  uint32_t gwords[kChunkTiles][kGroups];
  uint32_t gmeta[kChunkTiles][kGroups];
  uint32_t chunk;                     // chunk id or kSentinel
  uint32_t ntiles;
};

// FB = bytes of fixed-length (F) bytes staged per tile: 512 / 256 for
// L = 8 / 16 (one F per block, read by the lane that decodes the block)
template <int FB>
struct DecompressSmem {
  uint32_t data[kDStages][kDataWords];         // 25.7 KB
  uint2 ginfo[kDStages][kGroups];              // per 4-block group: {words per block (bytes), offset | mode << 16}
  uint32_t tile[kDStages];
  uint32_t delta[kDStages];                    // first payload word of the tile inside data[]
  ChunkDesc chunk[2];
  alignas(16) uint32_t scratch[kComputeWarps][4 * 32];   // per-warp transposed rows of one group
  uint64_t full[kDStages];                     // TMA completion (the only mbarriers)
  alignas(16) uint8_t fbytes[kDStages][FB];
};

// named barriers (id 0 is __syncthreads)
constexpr uint32_t kBarEmpty0 = 1;
constexpr uint32_t kBarReady0 = kBarEmpty0 + kDStages, kBarFree0 = kBarReady0 + 2;
constexpr uint32_t kBarCount = 32 + 32 * kComputeWarps;   // loader + compute warps
static_assert(kBarFree0 + 2 <= 16, "named barriers");

// 8 x 8 bit-matrix transpose of hi:lo (bit p of byte i -> bit i of byte p),
// self-inverse: 8 planes of 8 elements -> the elements' bytes (a10 for
// L = 8 / 16; the compressor's transpose8x8)
__device__ __forceinline__ void untranspose8x8(uint32_t& lo, uint32_t& hi) {
  uint32_t t;
  t = (lo ^ (lo >> 7)) & 0x00AA00AAu;  lo ^= t ^ (t << 7);
  t = (hi ^ (hi >> 7)) & 0x00AA00AAu;  hi ^= t ^ (t << 7);
  t = (lo ^ (lo >> 14)) & 0x0000CCCCu; lo ^= t ^ (t << 14);
  t = (hi ^ (hi >> 14)) & 0x0000CCCCu; hi ^= t ^ (t << 14);
  t = (lo ^ __funnelshift_r(lo, hi, 28)) & 0xF0F0F0F0u;
  lo ^= t;
  hi ^= t >> 4;
}

// byte e of hi:lo -> byte g of v[e] (8 byte permutes)
template <int G>
__device__ __forceinline__ void scatter_bytes8(uint32_t lo, uint32_t hi, uint32_t* v) {
  constexpr uint32_t kKeep = 0x3210u & ~(0xFu << (4 * G));
#pragma unroll
  for (int e = 0; e < 8; ++e)
    v[e] = __byte_perm(v[e], e < 4 ? lo : hi, kKeep | ((4u + uint32_t(e & 3)) << (4 * G)));
}

// planes 8g .. 8g+7 of an L-block's byte sequence (kW = L/4 words) -> byte g
// of each element's v = 2|l| + s (inverse of the compressor's block_seq8)
template <int SL>
__device__ __forceinline__ void block_unseq8(const uint32_t* sq, int g, uint32_t* v) {
  auto put = [&](uint32_t lo, uint32_t hi, uint32_t* ve) {
    untranspose8x8(lo, hi);
    switch (g) {
      case 0: scatter_bytes8<0>(lo, hi, ve); break;
      case 1: scatter_bytes8<1>(lo, hi, ve); break;
      case 2: scatter_bytes8<2>(lo, hi, ve); break;
      default: scatter_bytes8<3>(lo, hi, ve); break;
    }
  };
  if constexpr (SL == 8) {
    put(sq[0], sq[1], v);
  } else {                                          // plane = [elements 0-7 byte, elements 8-15 byte]
    put(__byte_perm(sq[0], sq[1], 0x6420u), __byte_perm(sq[2], sq[3], 0x6420u), v);
    put(__byte_perm(sq[0], sq[1], 0x7531u), __byte_perm(sq[2], sq[3], 0x7531u), v + 8);
  }
}

}  // namespace

// M = L / 32: see compress.cu -- sub-block i of a block
// finds its word k at M k + i of the block's payload, and the in-block
// prefix sum (a11) runs over the block's M sub-blocks.
// D = Lorenzo dimensions (R18): 2 / 3 invert the block-local predictor of
// 1x4x8 / 2x4x4 blocks and scatter each block's rows into the (nz, ny, nx) field.
// CT = tiles per look-back chunk (4 or 8; 8 is instantiated for the main path
// only, chosen by the host for large inputs).
// SL = 8 / 16: byte-granular block lengths, one block per lane (M = 1).
template <int M, int O, int D = 1, int CT = 4, int SL = 0>
__global__ void __launch_bounds__(kDThreads, CUSZP_D_MINBLOCKS) decompress_kernel(DecompressArgs a) {
  static_assert(CT == 4 || CT == 8, "chunk of 4 or 8 tiles");
  static_assert(SL == 0 || ((SL == 8 || SL == 16) && M == 1 && O == 1 && D == 1), "L = 8 / 16");
  constexpr bool kSmall = SL != 0;
  constexpr int kFT = kSmall ? kTileElems / SL : 16;            // F bytes per tile (L = 8 / 16)
  static_assert(D == 1 || (M == 1 && O == 1), "multi-dimensional Lorenzo with L = 32, order 1");
  static_assert(M == 1 || M == 2 || M == 4, "L in {32, 64, 128}");
  static_assert(O == 1 || (O == 2 && M == 1), "2-layer Lorenzo with L = 32");
  constexpr uint32_t kLog2L = SL == 8 ? 3 : SL == 16 ? 4 : 5 + (M == 2 ? 1 : M == 4 ? 2 : 0);
  extern __shared__ __align__(128) unsigned char smem_raw[];
  DecompressSmem<kFT>& sm = *reinterpret_cast<DecompressSmem<kFT>*>(smem_raw);
  const int lane = threadIdx.x & 31;
  const int warp = __shfl_sync(0xffffffffu, int(threadIdx.x >> 5), 0);   // provably warp-uniform (no divergence checks before warp-sync ops)
  pdl_wait();                                     // compression / previous call complete
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
    if (magic != 0x505A5343u || h[4] != CUSZP_VERSION || h[7] != kLog2L ||
        ((h[5] & 0x10) != 0) != (O == 2) ||                 // predictor order (R17)
        ((h[5] >> 5) & 3) != D - 1)                          // predictor dimensions (R18)
      err = CUSZP_ECORRUPT;
    else if (h[6] != CUSZP_OK) err = (h[6] == CUSZP_ERANGE) ? CUSZP_ERANGE : CUSZP_ECORRUPT;
    else if (hn != a.n) err = CUSZP_EINVAL;
    else if (a.n > 0) {
      const float two = __fadd_rn(eb, eb);
      if (!(eb >= kFltMin) || !isfinite(two)) err = CUSZP_ECORRUPT;
      else if ((!kSmall && (pbytes & 3u)) || a.in_bytes < p0 || a.in_bytes - p0 < pbytes) err = CUSZP_ECORRUPT;
      payload_words = kSmall ? pbytes : pbytes / 4;        // look-back unit: bytes for L = 8 / 16
    }
  }
  const float two_eb = __fadd_rn(eb, eb);
  constexpr uint32_t ct = CT;
  const uint32_t num_chunks = (a.num_tiles + ct - 1) / ct;
  uint32_t bad = 0;

  if (threadIdx.x == 0) {
    for (int s = 0; s < kDStages; ++s) mbar_init(&sm.full[s], 1);
    fence_mbar_init();
  }
  __syncthreads();

  if (err == CUSZP_OK && a.n > 0) {
    if (warp == 0) {
      // ------------------------------------------------------------- scanner
      for (uint32_t i = 0;; ++i) {
        const int b = int(i & 1u);
        if (i >= 2) named_sync(kBarFree0 + b, 64);
        ChunkDesc& cd = sm.chunk[b];
        uint32_t c = 0;
        if (lane == 0) {
          stress_delay(i);
          c = atomicAdd(&a.ws->ticket, 1u);
        }
        c = __shfl_sync(kFull, c, 0);
        if (c >= num_chunks) {
          if (lane == 0) cd.chunk = kSentinel;
          named_arrive(kBarReady0 + b, 64);
          break;
        }
        const uint32_t t0 = c * ct;
        const uint32_t ntiles = min(ct, a.num_tiles - t0);
#ifdef CUSZP_TRACE
        if (a.trace && uint32_t(lane) < ntiles) trace_put(a.trace, t0 + lane, 0, global_ns());
#endif
        if constexpr (kSmall) {
          // L = 8 / 16: lane L sums the block bytes (Eq 2: (F + 1) L/8, 0 for
          // F = 0) of kSPL warp slices of the chunk (slice q = tile q / 8,
          // compute warp q % 8; 64 / 32 F bytes each, 16 per load).
          constexpr int kSlice = kFT / kComputeWarps;
          constexpr int kSPL = CT * kComputeWarps / 32;         // slices per lane: 2 (CT = 8) or 1
          constexpr int kLPT = kComputeWarps / kSPL;            // lanes per tile
          uint32_t ssum[kSPL], fmax = 0, lsum = 0;
#pragma unroll
          for (int h = 0; h < kSPL; ++h) {
            const uint32_t q = uint32_t(kSPL * lane + h);
            const uint64_t blk0 = uint64_t(t0 + q / 8) * kFT + (q % 8) * kSlice;
            uint4 f[kSlice / 16];
#pragma unroll
            for (int k = 0; k < kSlice / 16; ++k) {             // all loads in flight first
              const uint64_t bk = blk0 + 16 * k;
              f[k] = bk < a.nb ? *reinterpret_cast<const uint4*>(a.in + kHdr + bk) : make_uint4(0, 0, 0, 0);
            }
            uint32_t sum = 0;
#pragma unroll
            for (int k = 0; k < kSlice / 16; ++k) {
              const uint64_t bk = blk0 + 16 * k;
              uint32_t x[4] = {f[k].x, f[k].y, f[k].z, f[k].w};
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                if (bk + 4 * e + 4 > a.nb) {                    // the F area's padding: zero blocks
                  const int keep = int(a.nb > bk + 4 * e ? a.nb - bk - 4 * e : 0);
                  x[e] &= __funnelshift_rc(0xffffffffu, 0u, uint32_t(32 - 8 * keep));
                }
                fmax = __vmaxu4(fmax, x[e]);
                const uint32_t y = x[e] + (__vcmpne4(x[e], 0u) & 0x01010101u);   // F + 1 or 0 per byte
                sum += (y * 0x01010101u) >> 24;                 // <= 4 x 25
              }
            }
            ssum[h] = sum * uint32_t(SL / 8);
            lsum += ssum[h];
          }
          // tile-local exclusive slice offsets: segmented scan over a tile's lanes
          uint32_t incl = lsum;
#pragma unroll
          for (int o = 1; o < kLPT; o <<= 1) incl = uint32_t(scan_step_up(int(incl), o, (32 - kLPT) << 8));
          uint32_t ttot[CT], tpre[CT], agg = 0;
#pragma unroll
          for (int k = 0; k < CT; ++k) {
            ttot[k] = __shfl_sync(kFull, incl, kLPT * k + kLPT - 1);
            tpre[k] = agg;
            agg += ttot[k];
          }
          const bool badf = __any_sync(kFull, __vcmpgtu4(fmax, 0x18181818u) != 0u);   // F > 24
          if (lane == 0) publish_aggregate(a.status, c, agg, epoch);
          const uint64_t excl = resolve_prefix(a.status, c, agg, epoch);
          const bool oob = badf || excl + agg > payload_words;  // decode zeros, never read past in_bytes
          if (oob) bad |= kBadCorrupt;
          const int tl = lane / kLPT;
          uint32_t off = incl - lsum;
#pragma unroll
          for (int h = 0; h < kSPL; ++h) {
            cd.gmeta[tl][(kSPL * lane + h) % 8] = oob ? 0xffffffffu : off;   // 0xffffffff: a zero tile
            off += ssum[h];
          }
          uint64_t ts = 0;
          uint32_t tw = 0;
#pragma unroll
          for (int k = 0; k < CT; ++k)
            if (lane == k) { ts = excl + tpre[k]; tw = oob ? 0u : ttot[k]; }
          if (lane < CT) {
            cd.tile_start[lane] = ts;
            cd.tile_words[lane] = tw;
          }
          if (lane == 0) {
            cd.chunk = c;
            cd.ntiles = ntiles;
          }
          named_arrive(kBarReady0 + b, 64);
          continue;
        }
        // The chunk in parts of 4 tiles (ct / 4 of them): in part h, lane L takes
        // sub-blocks 16L .. 16L+15 of tiles 4h .. 4h+3 = groups 4(L%8) .. +3 of
        // tile 4h + L/8 = blocks (16L ..)/M.  All F loads of the chunk are
        // issued before any is used (one memory latency per chunk).
        constexpr int kParts = CT / 4;
        uint32_t fw[kParts][4];
        uint64_t blkp[kParts];
#pragma unroll
        for (int h = 0; h < kParts; ++h) {
          const uint64_t blk = (uint64_t(t0 + 4 * h) * kTileBlocks + 16u * lane) / M;
          blkp[h] = blk;
          fw[h][0] = fw[h][1] = fw[h][2] = fw[h][3] = 0;
          if (blk < a.nb) {                                              // in the 16-B padded F area
            if constexpr (M == 1) {
              const uint4 fq = *reinterpret_cast<const uint4*>(a.in + kHdr + blk);
              fw[h][0] = fq.x; fw[h][1] = fq.y; fw[h][2] = fq.z; fw[h][3] = fq.w;
            } else if constexpr (M == 2) {
              // F of blocks 2g, 2g+1 replicated onto sub-blocks (4g .. 4g+3)
              const uint2 fq = *reinterpret_cast<const uint2*>(a.in + kHdr + blk);
              fw[h][0] = __byte_perm(fq.x, 0, 0x1100u); fw[h][1] = __byte_perm(fq.x, 0, 0x3322u);
              fw[h][2] = __byte_perm(fq.y, 0, 0x1100u); fw[h][3] = __byte_perm(fq.y, 0, 0x3322u);
            } else {
              const uint32_t fq = *reinterpret_cast<const uint32_t*>(a.in + kHdr + blk);
              fw[h][0] = __byte_perm(fq, 0, 0x0000u); fw[h][1] = __byte_perm(fq, 0, 0x1111u);
              fw[h][2] = __byte_perm(fq, 0, 0x2222u); fw[h][3] = __byte_perm(fq, 0, 0x3333u);
            }
          }
        }
        uint32_t ttot[CT], agg = 0, tpre[CT];
        const int tl = lane >> 3;
#pragma unroll
        for (int h = 0; h < kParts; ++h) {
          const uint64_t blk = blkp[h];
          uint32_t gw[4], gspan[4], gsum[4], lsum = 0;
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            gw[g] = 0;
            gspan[g] = 0;
            gsum[g] = 0;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              uint32_t f = (fw[h][g] >> (8 * k)) & 0xffu;
              if (blk + (4 * g + k) / M >= a.nb) f = 0;
              if (f > uint32_t(kMaxF)) { bad |= kBadCorrupt; f = 0; }
              const uint32_t wq = f ? f + 1 : 0;             // Eq 2 in 4-byte words
              gw[g] |= wq << (8 * k);
              gspan[g] = max(gspan[g], wq);
              gsum[g] += wq;
            }
            lsum += gsum[g];
          }
          // tile-local exclusive offsets: segmented scan over the 8 lanes of each tile
          uint32_t incl = lsum;
          incl = uint32_t(scan_step_up(int(incl), 1, 24 << 8));
          incl = uint32_t(scan_step_up(int(incl), 2, 24 << 8));
          incl = uint32_t(scan_step_up(int(incl), 4, 24 << 8));
          uint32_t off = incl - lsum;
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            const uint32_t mode = gspan[g] <= 8 ? 0u : (gspan[g] <= 16 ? 1u : 2u);
            cd.gwords[4 * h + tl][4 * (lane & 7) + g] = gw[g];
            cd.gmeta[4 * h + tl][4 * (lane & 7) + g] = off | (mode << 16);
            off += gsum[g];
          }
          // tile totals and the chunk aggregate
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            ttot[4 * h + k] = __shfl_sync(kFull, incl, 8 * k + 7);
            tpre[4 * h + k] = agg;
            agg += ttot[4 * h + k];
          }
        }
        // a9: global synchronisation (decoupled look-back over chunks)
        if (lane == 0) publish_aggregate(a.status, c, agg, epoch);
#ifdef CUSZP_TRACE
        if (a.trace && uint32_t(lane) < ntiles) trace_put(a.trace, t0 + lane, 1, global_ns());
        uint32_t tr_nw = 0, tr_ns = 0;
        const uint64_t excl = resolve_prefix(a.status, c, agg, epoch, &tr_nw, &tr_ns);
        if (a.trace && uint32_t(lane) < ntiles) {
          trace_put(a.trace, t0 + lane, 2, global_ns());
          trace_put(a.trace, t0 + lane, 6, (uint64_t(tr_nw) << 32) | tr_ns);
        }
#else
        const uint64_t excl = resolve_prefix(a.status, c, agg, epoch);
#endif
        const bool oob = excl + agg > payload_words;   // corrupt offsets: decode zeros, never read past in_bytes
        if (oob) {
          bad |= kBadCorrupt;
#pragma unroll
          for (int h = 0; h < kParts; ++h)
#pragma unroll
            for (int g = 0; g < 4; ++g) cd.gwords[4 * h + tl][4 * (lane & 7) + g] = 0u;
        }
        uint64_t ts = 0;
        uint32_t tw = 0;
#pragma unroll
        for (int k = 0; k < CT; ++k)
          if (lane == k) { ts = excl + tpre[k]; tw = oob ? 0u : ttot[k]; }
        if (lane < CT) {
          cd.tile_start[lane] = ts;
          cd.tile_words[lane] = tw;
        }
        if (lane == 0) {
          cd.chunk = c;
          cd.ntiles = ntiles;
        }
        named_arrive(kBarReady0 + b, 64);
      }
    } else if (warp == 1) {
      // -------------------------------------------------------------- loader
      // Tile k goes to stage k % S once the compute warps released it (named
      // barrier EMPTY); the compute warps wait for its bytes on the stage's
      // mbarrier themselves (suspending try_wait), so up to S payload copies
      // are in flight and the loader never waits for a TMA to land.
      uint32_t k = 0;              // tiles loaded so far
      for (uint32_t i = 0;; ++i) {
        const int b = int(i & 1u);
        named_sync(kBarReady0 + b, 64);
        const ChunkDesc& cd = sm.chunk[b];
        if (cd.chunk == kSentinel) {
          const int s = int(k % kDStages);
          if (k >= uint32_t(kDStages)) named_sync(kBarEmpty0 + s, kBarCount);
          if (lane == 0) {
            sm.tile[s] = kSentinel;  // sync: mbarrier full[s]
            mbar_arrive(&sm.full[s]);
          }
          break;
        }
        for (uint32_t j = 0; j < cd.ntiles; ++j) {
          const int s = int(k % kDStages);
          if (k >= uint32_t(kDStages)) named_sync(kBarEmpty0 + s, kBarCount);
          sm.ginfo[s][lane] = make_uint2(cd.gwords[j][lane], cd.gmeta[j][lane]);  // sync: mbarrier full[s]; reused after the EMPTY named barrier
          const uint64_t tw = cd.tile_words[j];
          uint32_t tma_bytes = 0, delta = 0;
          uint64_t a0 = 0;
          if (tw > 0) {
            constexpr uint32_t kU = kSmall ? 1u : 4u;             // bytes per look-back unit
            const uint64_t start = p0 + kU * cd.tile_start[j], end = start + kU * tw;
            a0 = start & ~uint64_t(15);
            uint64_t a1 = (end + 15) & ~uint64_t(15);
            if (a1 > a.in_bytes) a1 = a.in_bytes & ~uint64_t(15);
            tma_bytes = uint32_t(a1 - a0);
            delta = uint32_t(start - a0) / kU;
            if constexpr (kSmall) {
              // bytes past the last full 16 bytes inside in_bytes (<= 15)
              const uint64_t tail = end > a1 ? end - a1 : 0;
              if (uint64_t(lane) < tail)
                reinterpret_cast<uint8_t*>(sm.data[s])[(a1 - a0) + lane] = a.in[a1 + lane];  // sync: mbarrier full[s]
            } else {
              // words past the last full 16 bytes inside in_bytes (<= 3)
              const uint64_t tail_words = end > a1 ? (end - a1) / 4 : 0;
              if (uint64_t(lane) < tail_words)
                sm.data[s][(a1 - a0) / 4 + lane] = *reinterpret_cast<const uint32_t*>(a.in + a1 + 4 * lane);  // sync: mbarrier full[s]
            }
          }
          __syncwarp();
          if (lane == 0) {
            sm.tile[s] = cd.chunk * ct + j;  // sync: mbarrier full[s]
            sm.delta[s] = delta;  // sync: mbarrier full[s]
            // L = 8 / 16: the tile's F bytes too (the decoding lanes read them)
            const uint32_t t_ld = cd.chunk * ct + j;
            const uint32_t fb = kSmall ? uint32_t(min(uint64_t(kFT), align16(a.nb) - uint64_t(t_ld) * kFT)) : 0u;
            mbar_arrive_expect_tx(&sm.full[s], tma_bytes + fb);   // one phase per use, even with 0 bytes
            if (tma_bytes) tma_load_1d(sm.data[s], a.in + a0, tma_bytes, &sm.full[s]);
            if (kSmall) tma_load_1d(sm.fbytes[s], a.in + kHdr + uint64_t(t_ld) * kFT, fb, &sm.full[s]);
#ifdef CUSZP_TRACE
            trace_put(a.trace, cd.chunk * ct + j, 3, global_ns());
            trace_put(a.trace, cd.chunk * ct + j, 7, blockIdx.x);
#endif
          }
          ++k;
        }
        named_arrive(kBarFree0 + b, 64);
      }
    } else if constexpr (kSmall) {
      // ------------------------------------------- compute, L = 8 / 16
      // One block per lane (kBPL passes of 32 blocks per tile): the lane's F
      // byte gives its planes (F + 1, 0 for a zero block) and bytes (Eq 2); a
      // warp scan plus the scanner's slice offset places the block in the
      // staged payload; its byte sequence is read as funnel-shifted words
      // (bytes past the block masked off), 8 planes at a time turned back
      // into element bytes by the self-inverse 8x8 bit transpose (a10), then
      // the in-register prefix sum (a11) and dequantisation (a12).
      const int w = warp - kDFirstCompute;
      constexpr int kSlice = kFT / kComputeWarps;
      constexpr int kBPL = kSlice / 32;                            // 2 (L = 8), 1 (L = 16)
      constexpr int kW = SL / 4;                                    // sequence words per 8 planes
      const float two_eb_s = __fmul_rn(two_eb, 0x1p23f);
      const bool scaled_ok = isfinite(two_eb_s);
      for (uint32_t i = 0;; ++i) {
        const int s = int(i % kDStages);
        mbar_wait(&sm.full[s], (i / kDStages) & 1u);            // payload + F bytes landed
        const uint32_t t = sm.tile[s];  // sync: mbarrier full[s]
        if (t == kSentinel) break;
        const uint32_t so_raw = sm.ginfo[s][w].y;  // sync: mbarrier full[s]
        const bool zero_tile = so_raw == 0xffffffffu;
        uint32_t base = sm.delta[s] + (zero_tile ? 0u : so_raw);  // sync: mbarrier full[s]
#pragma unroll 1
        for (int p = 0; p < kBPL; ++p) {
          const uint32_t blk = uint32_t(p * 32 + lane);                // block in the warp's slice
          const uint64_t gblk = uint64_t(t) * kFT + uint64_t(w) * kSlice + blk;
          uint32_t F = sm.fbytes[s][w * kSlice + blk];  // sync: mbarrier full[s]
          if (gblk >= a.nb || zero_tile || F > uint32_t(kMaxF)) F = 0;
          const uint32_t planes = F ? F + 1 : 0u, c = planes * uint32_t(SL / 8);
          uint32_t incl = c;
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(kFull, incl, d);
            if (lane >= d) incl += y;
          }
          const uint32_t off = base + incl - c;                      // byte offset in data[s]
          base += __shfl_sync(kFull, incl, 31);
          const uint32_t G = (__reduce_max_sync(kFull, planes) + 7) >> 3;
          const uint32_t* dw = sm.data[s] + (off >> 2);
          const uint32_t sh = 8 * (off & 3u);
          uint32_t v[SL];
#pragma unroll
          for (int e = 0; e < SL; ++e) v[e] = 0;
          uint32_t wprev = dw[0];  // sync: mbarrier full[s]
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            if (uint32_t(g) < G) {
              uint32_t sq[kW];
#pragma unroll
              for (int k = 0; k < kW; ++k) {
                const int j = g * kW + k;
                const uint32_t wn = dw[j + 1];  // sync: mbarrier full[s]
                const int rem = int(c) - 4 * j;                      // bytes of the block left
                sq[k] = __funnelshift_r(wprev, wn, sh) &
                        __funnelshift_rc(0xffffffffu, 0u, uint32_t(min(max(32 - 8 * rem, 0), 32)));
                wprev = wn;
              }
              block_unseq8<SL>(sq, g, v);
            }
          }
          float* o = a.out + uint64_t(t) * kTileElems + uint64_t(w) * (kSlice * SL) + uint64_t(blk) * SL;
          float d[SL];
          if (scaled_ok) {
            // v rotated right by one = sign | |l|: the subnormal l * 2^-149;
            // the running sum is exact (|r| < 2^23), then (r 2^-149 * 2^126) *
            // (2eb * 2^23) is the single rounding of r * 2eb (R13)
            float r = 0.0f;
#pragma unroll
            for (int e = 0; e < SL; ++e) {
              r = __fadd_rn(r, __uint_as_float(__funnelshift_r(v[e], v[e], 1)));
              d[e] = __fmul_rn(__fmul_rn(r, 0x1p126f), two_eb_s);
            }
          } else {
            int r = 0;
#pragma unroll
            for (int e = 0; e < SL; ++e) {
              r += (v[e] & 1u) ? -int(v[e] >> 1) : int(v[e] >> 1);
              d[e] = __fmul_rn(__int2float_rn(r), two_eb);
            }
          }
          const uint64_t i0 = uint64_t(o - a.out);
          if (i0 + SL <= a.n) {
#pragma unroll
            for (int q = 0; q < SL / 4; ++q)
              reinterpret_cast<float4*>(o)[q] = make_float4(d[4 * q], d[4 * q + 1], d[4 * q + 2], d[4 * q + 3]);
          } else {
#pragma unroll
            for (int e = 0; e < SL; ++e)
              if (i0 + e < a.n) o[e] = d[e];
          }
        }
        named_arrive(kBarEmpty0 + s, kBarCount);
      }
    } else {
      // ------------------------------------------------------------ compute
      const int w = warp - kDFirstCompute;
      const Xpose xpose(lane);
      // scaled-float inverse Lorenzo (order 1, any L): 2eb * 2^23 must be finite,
      // else (2eb >= 2^105, absurd bounds) the integer path runs
      const float two_eb_s = __fmul_rn(two_eb, 0x1p23f);
      const bool scaled_ok = isfinite(two_eb_s);
      const uint64_t two_eb_s2 = (uint64_t(__float_as_uint(two_eb_s)) << 32) | __float_as_uint(two_eb_s);
      constexpr uint64_t kUp126x2 = 0x7E8000007E800000ull;          // 2^126, twice
      uint32_t* scratch = sm.scratch[w];
      // per-lane constants: quad mode -> block q = lane/8 owns lanes 8q..8q+7;
      // pair mode -> blocks (0,1) in lanes 0-15 / 16-31 of row 0, (2,3) of row 1
      const uint32_t q = uint32_t(lane) >> 3, k8 = lane & 7, k16 = lane & 15;
      const bool hi = lane >= 16;
      const uint32_t sel_quad = 0x4440u + q;                        // PRMT: byte q, zero-extended
      const uint32_t sel_pair = (q & 1) ? 0x4432u : 0x4410u;        // PRMT: half q&1, zero-extended
      const uint32_t row_pair = (q >> 1) * 32u, row_single = q * 32u;
      const uint32_t sel_b01 = hi ? 0x4441u : 0x4440u, sel_b23 = hi ? 0x4443u : 0x4442u;
      const uint32_t lane4 = 4u * k8;
      auto compute_role = [&](auto scaled_tag) {
      constexpr bool kScaledD = decltype(scaled_tag)::value;
      for (uint32_t i = 0;; ++i) {
        const int s = int(i % kDStages);
        mbar_wait(&sm.full[s], (i / kDStages) & 1u);          // tile's payload landed (suspending wait)
        const uint32_t t = sm.tile[s];  // sync: mbarrier full[s]
        if (t == kSentinel) break;
#ifdef CUSZP_TRACE
        if (a.trace && lane == 0) {
          const uint64_t now = global_ns();
          if (w == 0) trace_put(a.trace, t, 4, now);
          a.trace[16ull * a.num_tiles + 8ull * t + w] = now;          // per-warp pickup time
        }
#endif
        const bool last = (t == a.num_tiles - 1);
        const uint32_t* data = sm.data[s] + sm.delta[s];  // sync: mbarrier full[s]
        float* outp = a.out + uint64_t(t) * kTileElems + uint64_t(w) * kBPW * 32 + q * 32u + lane4;
#pragma unroll kDUnroll
#ifdef CUSZP_DIAG_NOWORK
        for (int g = 0; g < 0; ++g) {   // diagnostics only: pipeline without the decode work
#else
        for (int g = 0; g < kBPW / 4; ++g) {
#endif
          const uint2 gi = sm.ginfo[s][w * 4 + g];  // sync: mbarrier full[s]
          const uint32_t wbytes = gi.x;
          const uint32_t* gdata = data + (gi.y & 0xffffu);
          const uint32_t mode = gi.y >> 16;
          const uint32_t pbytes = wbytes * 0x01010100u;             // exclusive word prefix per block
          uint32_t sel, row;                                         // phase-2 source of this lane
          // a10: load each packed block's words into its lane range, one transpose per row
          if (M > 1 && mode == 0) {
            // word k8 of sub-block q at pre(block) + M k8 + q % M
            const uint32_t wq = __byte_perm(wbytes, 0, sel_quad);
            const uint32_t pq = __byte_perm(pbytes, 0, 0x4440u + (q & ~uint32_t(M - 1))) + M * k8 + (q & (M - 1));
            scratch[lane] = xpose(k8 < wq ? gdata[pq] : 0u);
            sel = sel_quad;
            row = 0;
          } else if (M > 1 && mode == 1) {
            const uint32_t w0 = wbytes & 0xffu, w2 = (wbytes >> 16) & 0xffu;
            const uint32_t h = hi ? 1u : 0u;
            const uint32_t x01 = k16 < w0 ? gdata[M * k16 + h] : 0u;
            const uint32_t x23 = k16 < w2 ? gdata[(M == 2 ? 2 * w0 : 0u) + M * k16 + (M == 2 ? h : 2u + h)] : 0u;
            scratch[lane] = xpose(x01);
            scratch[32 + lane] = xpose(x23);
            sel = sel_pair;
            row = row_pair;
          } else if (M > 1) {
#pragma unroll
            for (int b = 0; b < 4; ++b) {
              const uint32_t wq = (wbytes >> (8 * b)) & 0xffu;
              const uint32_t oq = ((pbytes >> (8 * (b & ~(M - 1)))) & 0xffu) + (b & (M - 1));
              scratch[32 * b + lane] = xpose(uint32_t(lane) < wq ? gdata[oq + M * uint32_t(lane)] : 0u);
            }
            sel = 0x3210u;
            row = row_single;
          } else if (mode == 0) {
            const uint32_t wq = __byte_perm(wbytes, 0, sel_quad), pq = __byte_perm(pbytes, 0, sel_quad);
            scratch[lane] = xpose(k8 < wq ? gdata[pq + k8] : 0u);
            sel = sel_quad;
            row = 0;
          } else if (mode == 1) {
            // lanes 0-15 take blocks 0 / 2, lanes 16-31 blocks 1 / 3: word counts
            // and exclusive word offsets by per-lane byte selects
            const uint32_t x01 = k16 < __byte_perm(wbytes, 0, sel_b01) ? gdata[__byte_perm(pbytes, 0, sel_b01) + k16] : 0u;
            const uint32_t x23 = k16 < __byte_perm(wbytes, 0, sel_b23) ? gdata[__byte_perm(pbytes, 0, sel_b23) + k16] : 0u;
            scratch[lane] = xpose(x01);
            scratch[32 + lane] = xpose(x23);
            sel = sel_pair;
            row = row_pair;
          } else {
#pragma unroll
            for (int b = 0; b < 4; ++b) {
              const uint32_t wq = (wbytes >> (8 * b)) & 0xffu, oq = (pbytes >> (8 * b)) & 0xffu;
              scratch[32 * b + lane] = xpose(uint32_t(lane) < wq ? gdata[oq + lane] : 0u);
            }
            sel = 0x3210u;
            row = row_single;
          }
          __syncwarp();
          const uint4 raw = *reinterpret_cast<const uint4*>(&scratch[row + lane4]);
          constexpr int kSeg = (32 - 8 * M) << 8;                     // segment = the block's 8 M lanes
          if constexpr (kScaledD) {
            // v = 2|l| + s rotated right by one is sign | |l|: the bits of the
            // subnormal float l * 2^-149 (the encoder's
            // quantize_scaled2 in reverse).  Every sum the inverse Lorenzo
            // forms is r_b - r_a of one block, |.| < 2^23 under the R5
            // guard, so it stays on the subnormal grid and every add is
            // exact integer arithmetic.
            float f0 = __uint_as_float(__funnelshift_r(__byte_perm(raw.x, 0, sel), __byte_perm(raw.x, 0, sel), 1));
            float f1 = __uint_as_float(__funnelshift_r(__byte_perm(raw.y, 0, sel), __byte_perm(raw.y, 0, sel), 1));
            float f2 = __uint_as_float(__funnelshift_r(__byte_perm(raw.z, 0, sel), __byte_perm(raw.z, 0, sel), 1));
            float f3 = __uint_as_float(__funnelshift_r(__byte_perm(raw.w, 0, sel), __byte_perm(raw.w, 0, sel), 1));
            // a11: r_j = sum_{i <= j} l_i within the block
            f1 = __fadd_rn(f1, f0);
            f2 = __fadd_rn(f2, f1);
            f3 = __fadd_rn(f3, f2);
            float incl = f3;
            incl = scan_step_up_f(incl, 1, kSeg);
            incl = scan_step_up_f(incl, 2, kSeg);
            incl = scan_step_up_f(incl, 4, kSeg);
            if constexpr (M >= 2) incl = scan_step_up_f(incl, 8, kSeg);
            if constexpr (M >= 4) incl = scan_step_up_f(incl, 16, kSeg);
            const float carry = __fsub_rn(incl, f3);                  // exact (same grid)
            // a12: d' = r * 2eb = (r 2^-149 * 2^126) * (2eb * 2^23): the first
            // product is exact (r 2^-23, a normal number), so the second is
            // the single rounding of r * 2eb -- bit-identical to R13.  Pairs
            // on the packed fp32 pipe (same RN semantics per element).
            uint64_t p01, p23, d01, d23;
            asm("mov.b64 %0, {%1, %2};" : "=l"(p01) : "f"(f0), "f"(f1));
            asm("mov.b64 %0, {%1, %2};" : "=l"(p23) : "f"(__fadd_rn(f2, carry)), "f"(incl));
            const uint64_t cc = (uint64_t(__float_as_uint(carry)) << 32) | __float_as_uint(carry);
            asm("add.rn.f32x2 %0, %0, %1;" : "+l"(p01) : "l"(cc));
            asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d01) : "l"(p01), "l"(kUp126x2));
            asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d23) : "l"(p23), "l"(kUp126x2));
            asm("mul.rn.f32x2 %0, %0, %1;" : "+l"(d01) : "l"(two_eb_s2));
            asm("mul.rn.f32x2 %0, %0, %1;" : "+l"(d23) : "l"(two_eb_s2));
            float4 d;
            asm("mov.b64 {%0, %1}, %2;" : "=f"(d.x), "=f"(d.y) : "l"(d01));
            asm("mov.b64 {%0, %1}, %2;" : "=f"(d.z), "=f"(d.w) : "l"(d23));
            float* o = outp + g * 128;
            if (!last) {
              *reinterpret_cast<float4*>(o) = d;
            } else {
              const uint64_t i0 = uint64_t(o - a.out);
              if (i0 + 4 <= a.n) *reinterpret_cast<float4*>(o) = d;
              else {
                if (i0 < a.n) o[0] = d.x;
                if (i0 + 1 < a.n) o[1] = d.y;
                if (i0 + 2 < a.n) o[2] = d.z;
              }
            }
            __syncwarp();
            continue;
          }
          // sign-magnitude v = 2|l| + s -> l
          int e0, e1, e2, e3;
          {
            const uint32_t v0 = __byte_perm(raw.x, 0, sel), v1 = __byte_perm(raw.y, 0, sel);
            const uint32_t v2 = __byte_perm(raw.z, 0, sel), v3 = __byte_perm(raw.w, 0, sel);
            e0 = (v0 & 1u) ? -int(v0 >> 1) : int(v0 >> 1);
            e1 = (v1 & 1u) ? -int(v1 >> 1) : int(v1 >> 1);
            e2 = (v2 & 1u) ? -int(v2 >> 1) : int(v2 >> 1);
            e3 = (v3 & 1u) ? -int(v3 >> 1) : int(v3 >> 1);
          }
          if constexpr (D > 1) {
            // R18: r = cumulative sums of l along x, y (and z) of the block.
            // This lane holds elements 4 k8 .. 4 k8 + 3 of block q: 2D row
            // k8/2, x = 4 (k8 % 2) + e; 3D plane k8/4, row k8 % 4, x = e.
            const uint32_t k8 = lane & 7u;
            constexpr int kSeg8 = 24 << 8;
            [[maybe_unused]] constexpr int kSeg4 = 28 << 8;
            e1 += e0;                                                 // along x, inside the lane
            e2 += e1;
            e3 += e2;
            if constexpr (D == 2) {
              const int cx = __shfl_up_sync(kFull, e3, 1);            // the row's left half
              if (k8 & 1u) { e0 += cx; e1 += cx; e2 += cx; e3 += cx; }
              e0 = scan_step_up(e0, 2, kSeg8); e1 = scan_step_up(e1, 2, kSeg8);   // along y (lanes 2 apart)
              e2 = scan_step_up(e2, 2, kSeg8); e3 = scan_step_up(e3, 2, kSeg8);
              e0 = scan_step_up(e0, 4, kSeg8); e1 = scan_step_up(e1, 4, kSeg8);
              e2 = scan_step_up(e2, 4, kSeg8); e3 = scan_step_up(e3, 4, kSeg8);
            } else {
              e0 = scan_step_up(e0, 1, kSeg4); e1 = scan_step_up(e1, 1, kSeg4);   // along y (4-lane planes)
              e2 = scan_step_up(e2, 1, kSeg4); e3 = scan_step_up(e3, 1, kSeg4);
              e0 = scan_step_up(e0, 2, kSeg4); e1 = scan_step_up(e1, 2, kSeg4);
              e2 = scan_step_up(e2, 2, kSeg4); e3 = scan_step_up(e3, 2, kSeg4);
              e0 = scan_step_up(e0, 4, kSeg8); e1 = scan_step_up(e1, 4, kSeg8);   // along z
              e2 = scan_step_up(e2, 4, kSeg8); e3 = scan_step_up(e3, 4, kSeg8);
            }
            float dd[4];
            dd[0] = __fmul_rn(__int2float_rn(e0), two_eb);           // a12 (R13)
            dd[1] = __fmul_rn(__int2float_rn(e1), two_eb);
            dd[2] = __fmul_rn(__int2float_rn(e2), two_eb);
            dd[3] = __fmul_rn(__int2float_rn(e3), two_eb);
            const uint32_t b = t * uint32_t(kTileBlocks) + uint32_t(w) * kBPW + uint32_t(g) * 4u + q;
            const uint32_t kyz = a.fd_nbx.div(b), kx = b - kyz * uint32_t(a.nbx);   // FastDiv (internal.cuh)
            const uint32_t kz = a.fd_nby.div(kyz), ky = kyz - kz * uint32_t(a.nby);
            uint64_t gz, gy, gx;
            if constexpr (D == 2) { gz = kz; gy = ky * 4u + (k8 >> 1); gx = kx * 8u + 4u * (k8 & 1u); }
            else { gz = kz * 2u + (k8 >> 2); gy = ky * 4u + (k8 & 3u); gx = kx * 4u; }
            if (b < a.nb && gz < a.nz && gy < a.ny) {
              float* o = a.out + (gz * a.ny + gy) * a.nx + gx;
              if (gx + 4 <= a.nx && (reinterpret_cast<uintptr_t>(o) & 15u) == 0) {
                *reinterpret_cast<float4*>(o) = make_float4(dd[0], dd[1], dd[2], dd[3]);
              } else {
#pragma unroll
                for (int e = 0; e < 4; ++e)
                  if (gx + e < a.nx) o[e] = dd[e];
              }
            }
            __syncwarp();
            continue;
          }
          // a11: r_j = sum_{i <= j} l_i within the block
          e1 += e0;
          e2 += e1;
          e3 += e2;
          int incl = e3;
          incl = scan_step_up(incl, 1, kSeg);
          incl = scan_step_up(incl, 2, kSeg);
          incl = scan_step_up(incl, 4, kSeg);
          if constexpr (M >= 2) incl = scan_step_up(incl, 8, kSeg);
          if constexpr (M >= 4) incl = scan_step_up(incl, 16, kSeg);
          const int carry = incl - e3;
          e0 += carry;
          e1 += carry;
          e2 += carry;
          e3 = incl;
          if constexpr (O == 2) {
            // 2-layer Lorenzo (R17): the first prefix sum gave r_j - r_{j-1};
            // a second one over the block gives r_j
            e1 += e0;
            e2 += e1;
            e3 += e2;
            int inc2 = e3;
            inc2 = scan_step_up(inc2, 1, kSeg);
            inc2 = scan_step_up(inc2, 2, kSeg);
            inc2 = scan_step_up(inc2, 4, kSeg);
            const int c2 = inc2 - e3;
            e0 += c2;
            e1 += c2;
            e2 += c2;
            e3 = inc2;
          }
          // a12: d' = r * 2eb
          float4 d;
          d.x = __fmul_rn(__int2float_rn(e0), two_eb);
          d.y = __fmul_rn(__int2float_rn(e1), two_eb);
          d.z = __fmul_rn(__int2float_rn(e2), two_eb);
          d.w = __fmul_rn(__int2float_rn(e3), two_eb);
          float* o = outp + g * 128;
          if (!last) {
            *reinterpret_cast<float4*>(o) = d;
          } else {
            const uint64_t i0 = uint64_t(o - a.out);
            if (i0 + 4 <= a.n) *reinterpret_cast<float4*>(o) = d;
            else {
              if (i0 < a.n) o[0] = d.x;
              if (i0 + 1 < a.n) o[1] = d.y;
              if (i0 + 2 < a.n) o[2] = d.z;
            }
          }
          __syncwarp();
        }
#ifdef CUSZP_TRACE
        if (a.trace && lane == 0) {
          const uint64_t now = global_ns();
          a.trace[8ull * a.num_tiles + 8ull * t + w] = now;          // per-warp done time
          atomicMax(reinterpret_cast<unsigned long long*>(a.trace + 8ull * t + 5), now);
        }
#endif
        named_arrive(kBarEmpty0 + s, kBarCount);
      }
      };
      // one branch for the whole launch, not one per group
      if constexpr (D == 1 && O == 1) {
        if (scaled_ok) compute_role(std::true_type{});
        else compute_role(std::false_type{});
      } else {
        compute_role(std::false_type{});
      }
    }
  }

  if (cta_finish(a.ws, bad)) {
    uint32_t final_status = err;
    if (threadIdx.x == 0 && final_status == CUSZP_OK) {
      const uint32_t acc = *reinterpret_cast<volatile uint32_t*>(&a.ws->status_accum);
      if (acc & kBadCorrupt) final_status = CUSZP_ECORRUPT;
      if (final_status == CUSZP_OK && num_chunks > 0 && a.n > 0) {
        const uint64_t total = ld_relaxed_u64(a.status + num_chunks - 1) & kValueMask;
        if (total != payload_words) final_status = CUSZP_ECORRUPT;
      }
    }
    finish_call(a.ws, a.status, a.status_cap, epoch, final_status);
  }
}

namespace {
template <int M, int O = 1, int D = 1, int CT = 4, int SL = 0>
cudaError_t configure_m(int* occ) {
  constexpr int kFT = SL ? kTileElems / SL : 16;
  const int smem = int(sizeof(DecompressSmem<kFT>));
  cudaError_t e = cudaFuncSetAttribute(decompress_kernel<M, O, D, CT, SL>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, decompress_kernel<M, O, D, CT, SL>, kDThreads, smem);
  return e;
}
template <int M, int O = 1, int D = 1, int CT = 4, int SL = 0>
cudaError_t launch_k(cudaLaunchConfig_t cfg, const DecompressArgs& a) {
  constexpr int kFT = SL ? kTileElems / SL : 16;
  cfg.dynamicSmemBytes = sizeof(DecompressSmem<kFT>);
  return cudaLaunchKernelEx(&cfg, decompress_kernel<M, O, D, CT, SL>, a);
}
}  // namespace

// L in {8, 16, 32, 64, 128}: resident CTAs per SM of that block length's kernel
cudaError_t decompress_configure(int L, int* occ) {
  int occ2 = 0;
  if (L == 32 && (configure_m<1, 2>(&occ2) != cudaSuccess || configure_m<1, 1, 2>(&occ2) != cudaSuccess ||
                  configure_m<1, 1, 3>(&occ2) != cudaSuccess || configure_m<1, 1, 1, 8>(&occ2) != cudaSuccess))
    return cudaErrorUnknown;
  if (L == 8 && configure_m<1, 1, 1, 8, 8>(&occ2) != cudaSuccess) return cudaErrorUnknown;
  if (L == 16 && configure_m<1, 1, 1, 8, 16>(&occ2) != cudaSuccess) return cudaErrorUnknown;
  switch (L) {
    case 8: return configure_m<1, 1, 1, 4, 8>(occ);
    case 16: return configure_m<1, 1, 1, 4, 16>(occ);
    case 32: return configure_m<1>(occ);
    case 64: return configure_m<2>(occ);
    default: return configure_m<4>(occ);
  }
}

cudaError_t decompress_launch(int L, int order, unsigned grid, const DecompressArgs& a, cudaStream_t s) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kDThreads);
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;   // see pdl_wait()
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  const bool c8 = a.chunk_tiles == 8;
  if (a.dims == 2) return launch_k<1, 1, 2>(cfg, a);
  if (a.dims == 3) return launch_k<1, 1, 3>(cfg, a);
  if (order == 2) return launch_k<1, 2>(cfg, a);
  switch (L) {
    case 8: return c8 ? launch_k<1, 1, 1, 8, 8>(cfg, a) : launch_k<1, 1, 1, 4, 8>(cfg, a);
    case 16: return c8 ? launch_k<1, 1, 1, 8, 16>(cfg, a) : launch_k<1, 1, 1, 4, 16>(cfg, a);
    case 32: return c8 ? launch_k<1, 1, 1, 8>(cfg, a) : launch_k<1, 1>(cfg, a);
    case 64: return launch_k<2, 1>(cfg, a);
    default: return launch_k<4, 1>(cfg, a);
  }
}

size_t decompress_smem_bytes() { return sizeof(DecompressSmem<16>); }
int decompress_threads() { return kDThreads; }

}  // namespace cuszp
