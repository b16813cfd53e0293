// compress.cu -- the fused cuSZp compression kernel for sm_100a
// (paper sec 3.1 / Fig 2 and sec 4).
//
// Persistent, warp-specialised CTA:
//   warp 0      producer: takes a tile ticket, streams the tile's 16 KB of
//               fp32 HBM -> shared memory with one 1D TMA bulk copy
//               (UBLKCP) into a kStages-deep mbarrier ring;
//   warps 1..kWriters  writers (below);
//   warps kWriters+1..  compute (kCW warps): 128/kCW L-blocks each, one lane per element:
//     a2 pre-quantisation   r = round(d / 2eb)            (R2)
//     a3 block Lorenzo      l_j = r_j - r_{j-1}, r_{-1}=0
//     a4 sign map + a8 bit-shuffle: v_j = 2|l_j| + [l_j<0]; a warp bit
//        transpose of v turns lane k into word k of the block: sign map
//        (k=0) then plane k-1 (R7, R9).  Two blocks
//        with F <= 15 share one transpose (bits 0-15 / 16-31).
//     a5 fixed length       words = bitlen(redux.max v) = F+1 (0: zero block)
//     a6 CmpL               4 * words bytes                 (Eq 2, R6)
//     payload words go to a shared-memory staging buffer, F bytes to HBM;
//     each compute warp appends its words to its own shared-memory ring;
//     the last compute warp to finish a tile publishes the tile aggregate
//     (a7, first half of the decoupled look-back) at once;
//   writers, tiles round-robin: resolve the tile's prefix by
//               look-back (a7, Eq 3), copy the ring segments to
//               their global offsets and release ring space in tile order.
//               Up to kMeta tiles wait for their prefix while the compute
//               warps keep going, so the look-back latency stays hidden.
//               A segment is copied as unrolled groups of four 32-word
//               chunks (immediate offsets, one uniform exit test per group).
// Paths that are rare on real fields -- the R2 redo of a group and a group
// with a block of more than 16 words -- are out-of-line calls, so the
// unrolled encode loop stays small (the instruction cache matters, DESIGN
// sec 8.1).
// Block lengths L = 64 / 128 (M = L/32 sub-blocks per block) reuse the L = 32
// encode; L = 8 / 16 (SL) encode one block per LANE (16 consecutive floats
// per lane: 2 blocks of 8 or 1 of 16) with in-register 8x8 bit transposes
// and byte-granular rings, look-back and copy-out.  D = 2 / 3
// (multi-dimensional Lorenzo, R18): the producer gathers blocks with cp.async.
#include "internal.cuh"

namespace cuszp {

namespace {

#ifndef CUSZP_C_STAGES
#define CUSZP_C_STAGES 2
#endif
#ifndef CUSZP_C_WRITERS
#define CUSZP_C_WRITERS 3
#endif
#ifndef CUSZP_C_META
#define CUSZP_C_META 8
#endif
#ifndef CUSZP_C_RING_WORDS
#define CUSZP_C_RING_WORDS 1024
#endif
#ifndef CUSZP_C_POLL_NS
#define CUSZP_C_POLL_NS 32
#endif
#ifndef CUSZP_C_LB_DELAY
#define CUSZP_C_LB_DELAY 1500   // ns before a writer's first look-back poll (tile still loading/encoding)
#endif
#ifndef CUSZP_C_CW
#define CUSZP_C_CW 8            // compute warps per CTA (each encodes 128 / CW blocks of a tile)
#endif
#ifndef CUSZP_C_MINBLOCKS
#define CUSZP_C_MINBLOCKS (CUSZP_C_CW > 8 ? 2 : 3)
#endif
#ifndef CUSZP_C_GUNROLL
#define CUSZP_C_GUNROLL 4
#endif
#ifndef CUSZP_C_L2_AHEAD
#define CUSZP_C_L2_AHEAD 1       // > 0: prefetch the input tile this many grids ahead into L2
#endif
#ifndef CUSZP_C_COPY_UNROLLED
#define CUSZP_C_COPY_UNROLLED 1  // copy-out of a ring segment in unrolled groups of 4 chunks (0: the round-2 loop)
#endif
#ifndef CUSZP_C_RARE_CALL
#define CUSZP_C_RARE_CALL 1      // the R2-correction redo and > 16-word stores of a group as out-of-line calls (L = 32, order 1)
#endif
#ifndef CUSZP_C_FULL_POLL_NS
#define CUSZP_C_FULL_POLL_NS 0   // > 0: compute warps poll their input stage with test + nanosleep
#endif
constexpr int kGUnroll = CUSZP_C_GUNROLL;         // groups of 4 blocks unrolled in the encode loop
constexpr int kStages = CUSZP_C_STAGES;          // input ring depth (16 KB tiles)
constexpr int kWriters = CUSZP_C_WRITERS;        // scan + writer warps
constexpr int kMeta = CUSZP_C_META;              // tiles between "computed" and "released"
constexpr uint32_t kRing = CUSZP_C_RING_WORDS;   // words per compute-warp ring (power of 2)
constexpr int kFirstCompute = 1 + kWriters;
constexpr int kTix = 16;                          // ticket ring: producer -> writers (early look-back)
static_assert(kStages + kMeta + kWriters <= kTix, "ticket ring");
constexpr int kCW = CUSZP_C_CW;                   // compute warps of this kernel
constexpr int kCBPW = kTileBlocks / kCW;          // 32-element blocks per compute warp per tile
static_assert(kCW == 8 || kCW == 16, "compute warps");
constexpr int kCThreads = (kFirstCompute + kCW) * 32;
static_assert((kRing & (kRing - 1)) == 0 && kRing >= 4 * 32, "ring size");

// WB = words of packed per-block plane counts per tile: 32 for L >= 32 (the
// 128 sub-blocks), 128 / 64 for L = 8 / 16 (512 / 256 blocks)
template <int WB>
struct alignas(16) TileMeta {
  uint32_t wb[WB];                 // plane counts (= F + 1, 0 for a zero block) of 4 blocks (bytes), tile order
  uint32_t tile;
  uint32_t agg;                    // words of the tile (bytes for L = 8 / 16)
  uint16_t cnt[kCW];               // words (bytes) per compute warp
  uint16_t head[kCW];              // ring position of each warp's first word (byte)
};

template <int WB>
struct CompressSmem {
  float in[kStages][kTileElems];                 // 32 KB
  uint32_t ring[kCW][kRing];                     // 4 KB per compute warp
  TileMeta<WB> meta[kMeta];
  uint32_t in_tile[kStages];
  uint32_t meta_done[kMeta];
  uint32_t tail[kCW];                            // ring words released (monotonic)
  uint32_t released;                             // CTA-local tiles released (monotonic)
  uint32_t tix[kTix];                            // tile of CTA-local tile j (slot j % kTix)
  uint64_t full[kStages], empty[kStages], staged[kMeta], tixbar[kTix];
};

__device__ __forceinline__ uint32_t ld_volatile_u32(const uint32_t* p) {
  return *reinterpret_cast<const volatile uint32_t*>(p);  // sync: flag poll (ring tail / released), ordered by the writer's fence
}

// R2 op sequence with explicit RN intrinsics (never contracted further):
// t = fma(d, recip, 1.5*2^23) rounds the exact product d*recip to the nearest
// integer (ties to even) in ONE rounding for |d*recip| < 2^22; r0 = t - 1.5*2^23
// is exact.  Returns the quantisation integer r BIASED by the magic's bit
// pattern (r + 0x4B400000), which the Lorenzo step removes for free.
//
// Fast path: r0.  It differs from round(d / 2eb) only when the exact residual
// |d - r0*2eb| exceeds eb (d/2eb within an ulp of a half integer), and
// NaN/Inf give a NaN residual: both set `rare`, and the group is then redone
// with the full correction (quantize_exact) -- the oracle's sequence in every
// case.  The R5 guard |r0| < 2^22 is tracked as a running max of |r0|.
// Two elements at once with the packed fp32 pipe (FFMA2 / FADD2; same IEEE
// RN semantics per element as the scalar sequence above).  Returns the two
// biased integers; updates the running max |r0| (guard) and max |res|.
__device__ __forceinline__ void quantize_fast2(float xa, float xb, float two_eb, float recip, float& rmax,
                                               float& resmax, uint32_t& ta, uint32_t& tb) {
  uint64_t x, t, r0, res;
  asm("mov.b64 %0, {%1, %2};" : "=l"(x) : "f"(xa), "f"(xb));
  const uint64_t rc = (uint64_t(__float_as_uint(recip)) << 32) | __float_as_uint(recip);
  const uint64_t mg = (uint64_t(__float_as_uint(kRoundMagic)) << 32) | __float_as_uint(kRoundMagic);
  const uint64_t nt = (uint64_t(__float_as_uint(-two_eb)) << 32) | __float_as_uint(-two_eb);
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(t) : "l"(x), "l"(rc), "l"(mg));
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r0) : "l"(t), "l"(mg));
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(res) : "l"(r0), "l"(nt), "l"(x));
  float r0a, r0b, ra, rb;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(r0a), "=f"(r0b) : "l"(r0));
  asm("mov.b64 {%0, %1}, %2;" : "=f"(ra), "=f"(rb) : "l"(res));
  asm("mov.b64 {%0, %1}, %2;" : "=r"(ta), "=r"(tb) : "l"(t));
  rmax = fmaxf(rmax, fmaxf(fabsf(r0a), fabsf(r0b)));       // R5 guard on finite values (Inf too)
  resmax = fmaxf(resmax, fmaxf(fabsf(ra), fabsf(rb)));
}

// M = 1, O = 1 fast path: the same R2 sequence, and the block Lorenzo step
// done on SCALED floats.  r0 * 2^-149 is the subnormal float whose bits are
// sign | |r0| (exact for |r0| < 2^23: the subnormal grid is the integer grid
// scaled by 2^-149), so the difference of two neighbours, computed exactly by
// one fma, has bits sign(l) | |l| for |l| < 2^23 (always, under the R5 guard)
// and a rotate left by one gives v = 2|l| + [l < 0] directly.  lane 0 takes
// r_{-1} = 0 through k = 0 in l = fma(prev, -k, r): prev * -0 + r = r
// (+0 for r = +0; r0 = t - magic is never -0).  Data failing the guard give
// garbage v, as on the integer path: such blocks are flagged ERANGE.
// Returns the two scaled values packed; updates rmax (|r0|) and resmax.
__device__ __forceinline__ uint64_t quantize_scaled2(float xa, float xb, float two_eb, float recip, float& rmax,
                                                     float& resmax) {
  uint64_t x, t, r0, res, rs;
  asm("mov.b64 %0, {%1, %2};" : "=l"(x) : "f"(xa), "f"(xb));
  const uint64_t rc = (uint64_t(__float_as_uint(recip)) << 32) | __float_as_uint(recip);
  const uint64_t mg = (uint64_t(__float_as_uint(kRoundMagic)) << 32) | __float_as_uint(kRoundMagic);
  const uint64_t nt = (uint64_t(__float_as_uint(-two_eb)) << 32) | __float_as_uint(-two_eb);
  const uint64_t sc = 0x0000000100000001ull;                  // 2^-149, the smallest subnormal, twice
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(t) : "l"(x), "l"(rc), "l"(mg));
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r0) : "l"(t), "l"(mg));
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(res) : "l"(r0), "l"(nt), "l"(x));
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(rs) : "l"(r0), "l"(sc));
  float r0a, r0b, ra, rb;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(r0a), "=f"(r0b) : "l"(r0));
  asm("mov.b64 {%0, %1}, %2;" : "=f"(ra), "=f"(rb) : "l"(res));
  rmax = fmaxf(rmax, fmaxf(fabsf(r0a), fabsf(r0b)));       // R5 guard on finite values (Inf too)
  resmax = fmaxf(resmax, fmaxf(fabsf(ra), fabsf(rb)));
  return rs;
}

// v for two rows at once: lanes j take the scaled r_{j-1} (lane 0: k = 0)
__device__ __forceinline__ void lorenzo_scaled2(uint64_t rs, uint64_t nk, uint32_t& va, uint32_t& vb) {
  uint32_t a, b;
  asm("mov.b64 {%0, %1}, %2;" : "=r"(a), "=r"(b) : "l"(rs));
  const uint32_t pa = __shfl_up_sync(kFull, a, 1), pb = __shfl_up_sync(kFull, b, 1);
  uint64_t p, l;
  asm("mov.b64 %0, {%1, %2};" : "=l"(p) : "r"(pa), "r"(pb));
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(l) : "l"(p), "l"(nk), "l"(rs));   // exact: r_j - r_{j-1}
  uint32_t la, lb;
  asm("mov.b64 {%0, %1}, %2;" : "=r"(la), "=r"(lb) : "l"(l));
  va = __funnelshift_l(la, la, 1);                             // sign | |l|  ->  2|l| + sign
  vb = __funnelshift_l(lb, lb, 1);
}

__device__ __forceinline__ uint32_t quantize_exact(float x, float eb, float two_eb, float recip, float& rmax) {
  const float t = __fmaf_rn(x, recip, kRoundMagic);
  const float r0 = __fsub_rn(t, kRoundMagic);
  if (!(fabsf(r0) < kGuard)) rmax = __int_as_float(0x7f800000);   // NaN too
  const float res = __fmaf_rn(-r0, two_eb, x);
  uint32_t r = __float_as_uint(t);
  r += uint32_t(int(res > eb) - int(res < -eb));
  return r;
}

// lane j holds the biased r_j of one block -> v_j = 2|l_j| + sign_j with the
// block Lorenzo l_j = r_j - r_{j-1}, r_{-1} = 0
__device__ __forceinline__ uint32_t lorenzo_pack(uint32_t rb, int lane) {
  uint32_t prev = __shfl_up_sync(kFull, rb, 1);
  prev = lane ? prev : kRoundMagicBits;
  const int l = int(rb - prev);
  const uint32_t a = uint32_t(l < 0 ? -l : l);
  return (a << 1) | (uint32_t(l) >> 31);
}
// The R2 correction of one group of 4 blocks (L = 32, order 1; 1D or the
// multi-dimensional predictors), out of line: the rare redo of the unrolled encode loop (an element within an ulp
// of a half integer of 2eb) as a call instead of four inlined copies, so the
// hot loop stays compact.  Returns v of the 4 blocks, their word counts
// (bytes of wb) and the updated guard maximum; 6 values, returned in
// registers.
struct RareOut { uint32_t v0, v1, v2, v3, wb; float vmax; };   // (rare_group_redo: after lorenzo_md_pack)

// same, lane 0 taking `first` (biased) as its predecessor: the last element
// of the previous 32-element sub-block of an L = 32 M block
__device__ __forceinline__ uint32_t lorenzo_pack_first(uint32_t rb, int lane, uint32_t first) {
  uint32_t prev = __shfl_up_sync(kFull, rb, 1);
  prev = lane ? prev : first;
  const int l = int(rb - prev);
  const uint32_t a = uint32_t(l < 0 ? -l : l);
  return (a << 1) | (uint32_t(l) >> 31);
}

// bit length of x (0 for x = 0): bfind gives the index of the highest set bit
// or 0xffffffff, so one add ends it (32 - clz compiles to FLO + two adds)
__device__ __forceinline__ uint32_t bitlen(uint32_t x) {
  uint32_t p;
  asm("bfind.u32 %0, %1;" : "=r"(p) : "r"(x));
  return p + 1u;
}

// a group with a block of more than 16 words (span > 16): one transpose per
// block, words appended to the ring at base (out of line: rare -- none of
// the bench fields has such a group at the bounds they are run at)
__device__ __noinline__ void store_singles(uint32_t* ring, uint32_t base, uint32_t v0, uint32_t v1, uint32_t v2,
                                           uint32_t v3, uint32_t wb, int lane) {
  const Xpose xpose(lane);
  const uint32_t v[4] = {v0, v1, v2, v3};
  uint32_t o = base;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const uint32_t tq = xpose(v[q]);
    const uint32_t wq = (wb >> (8 * q)) & 0xffu;
    if (uint32_t(lane) < wq) ring[(o + lane) & (kRing - 1)] = tq;  // sync: ring slot freed by the writer's tail release; read after staged[m]
    o += wq;
  }
}

// the virtual zero pad (R8) of the last tile's slice of one compute warp
// (kCBPW x 32 floats of the stage), then the proxy fence for the stage
template <int NPW>
__device__ __noinline__ void zero_tail_impl(float* src, uint64_t g0, uint64_t n, int lane) {
  for (int k = lane; k < NPW; k += 32)
    if (g0 + k >= n) src[k] = 0.0f;  // sync: own slice of the stage; no TMA rewrites it in this launch
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncwarp();
}

// bytes a, b, c, d (each < 256) -> one word, as 3 byte permutes
__device__ __forceinline__ uint32_t pack4(uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  return __byte_perm(__byte_perm(a, b, 0x3240u), __byte_perm(c, d, 0x3240u), 0x5410u);
}

}  // namespace

// M = L / 32: an L-block is M consecutive 32-element
// sub-blocks sharing one F; word k of sub-block i of a block sits at
// M k + i of the block's payload (a plane is L/8 bytes, element j at byte
// j/8, bit j%8 -- R9 generalised).  M = 1 is the paper's default L = 32.
// lane j holds the biased r_j of one block -> v_j for the 2-layer Lorenzo
// (R17): l_j = r_j - 2 r_{j-1} + r_{j-2}, r_{-1} = r_{-2} = 0
__device__ __forceinline__ uint32_t lorenzo2_pack(uint32_t rb, int lane) {
  uint32_t p1 = __shfl_up_sync(kFull, rb, 1), p2 = __shfl_up_sync(kFull, rb, 2);
  p1 = lane >= 1 ? p1 : kRoundMagicBits;
  p2 = lane >= 2 ? p2 : kRoundMagicBits;
  const int l = int(rb - p1) - int(p1 - p2);                 // the biases cancel
  const uint32_t a = uint32_t(l < 0 ? -l : l);
  return (a << 1) | (uint32_t(l) >> 31);
}

// lane j holds the biased r_j of one block in block order (element j =
// (z*4 + y)*bx + x) -> v_j for the block-local multi-dimensional Lorenzo
// (R18), as successive differences along x, y (and z), each taking 0 at the
// block's edge: 2D (4x8) l = r - r(x-1) - r(y-1) + r(y-1,x-1), 3D (2x4x4) the
// 7-term predictor.
template <int D>
__device__ __forceinline__ uint32_t lorenzo_md_pack(uint32_t rb, int lane) {
  constexpr int kBX = (D == 3) ? 4 : 8;
  uint32_t px = __shfl_up_sync(kFull, rb, 1);
  px = (lane % kBX) ? px : kRoundMagicBits;
  int l = int(rb - px);                                      // along x; the biases cancel
  const int uy = __shfl_up_sync(kFull, l, kBX);
  if ((lane / kBX) % 4) l -= uy;                             // along y
  if constexpr (D == 3) {
    const int uz = __shfl_up_sync(kFull, l, 16);
    if (lane >= 16) l -= uz;                                 // along z
  }
  const uint32_t a = uint32_t(l < 0 ? -l : l);
  return (a << 1) | (uint32_t(l) >> 31);
}

// ---------------------------------------------------------------- L = 8 / 16
// One L-block per LANE (thread-per-block): a plane of an L-block is L/8 BYTES
// (element j at byte j / 8, bit j % 8, R9 generalised), so the
// whole block -- quantisation, Lorenzo, fixed length and bit-shuffle -- runs
// in the lane's registers and no warp transpose is needed; only the block's
// byte offset comes from a warp scan.

// 8 x 8 bit-matrix transpose of the 64-bit value hi:lo (bit p of byte i ->
// bit i of byte p): bytes = the low / next ... byte of 8 elements -> 8 planes
// of those elements (the block bit-shuffle), three delta swaps
__device__ __forceinline__ void transpose8x8(uint32_t& lo, uint32_t& hi) {
  uint32_t t;
  t = (lo ^ (lo >> 7)) & 0x00AA00AAu;  lo ^= t ^ (t << 7);    // distance 7 and 14 stay inside
  t = (hi ^ (hi >> 7)) & 0x00AA00AAu;  hi ^= t ^ (t << 7);    // each 32-bit half
  t = (lo ^ (lo >> 14)) & 0x0000CCCCu; lo ^= t ^ (t << 14);
  t = (hi ^ (hi >> 14)) & 0x0000CCCCu; hi ^= t ^ (t << 14);
  t = (lo ^ __funnelshift_r(lo, hi, 28)) & 0xF0F0F0F0u;      // distance 28 crosses the halves
  lo ^= t;
  hi ^= t >> 4;
}

// byte g of 8 values -> one 64-bit row (byte i = value i's byte g)
__device__ __forceinline__ void gather_bytes8(const uint32_t* v, uint32_t g, uint32_t& lo, uint32_t& hi) {
  const uint32_t sel = g | ((4u + g) << 4);                     // PRMT: byte g of a, byte g of b
  lo = __byte_perm(__byte_perm(v[0], v[1], sel), __byte_perm(v[2], v[3], sel), 0x5410u);
  hi = __byte_perm(__byte_perm(v[4], v[5], sel), __byte_perm(v[6], v[7], sel), 0x5410u);
}

// Words 4q/W .. of an L-block's byte sequence for planes 8g .. 8g+7 (W = L/4
// words: the sign map is plane 0, then |l| bit k-1 in plane k)
template <int SL>
__device__ __forceinline__ void block_seq8(const uint32_t* v, uint32_t g, uint32_t* s) {
  uint32_t lo, hi;
  gather_bytes8(v, g, lo, hi);
  transpose8x8(lo, hi);
  if constexpr (SL == 8) {
    s[0] = lo;                                                  // planes 8g .. 8g+3, one byte each
    s[1] = hi;
  } else {                                                      // a plane = 2 bytes: elements 0-7, 8-15
    uint32_t lo1, hi1;
    gather_bytes8(v + 8, g, lo1, hi1);
    transpose8x8(lo1, hi1);
    s[0] = __byte_perm(lo, lo1, 0x5140u);
    s[1] = __byte_perm(lo, lo1, 0x7362u);
    s[2] = __byte_perm(hi, hi1, 0x5140u);
    s[3] = __byte_perm(hi, hi1, 0x7362u);
  }
}

// D = 1: the paper's block Lorenzo; D = 2 / 3: the block-local multi-
// dimensional predictor (R18), on the integer path like the inline redo
template <int D>
__device__ __noinline__ RareOut rare_group_redo(float x0, float x1, float x2, float x3, float eb, float two_eb,
                                                float recip, float vmax, int lane) {
  const float xs[4] = {x0, x1, x2, x3};
  uint32_t v[4], wb = 0;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const uint32_t r = quantize_exact(xs[q], eb, two_eb, recip, vmax);
    if constexpr (D == 1) v[q] = lorenzo_pack(r, lane);
    else v[q] = lorenzo_md_pack<D>(r, lane);
    wb |= bitlen(__reduce_or_sync(kFull, v[q])) << (8 * q);
  }
  return RareOut{v[0], v[1], v[2], v[3], wb, vmax};
}

// lorenzo_md_pack on SCALED values (quantize_scaled2's r 2^-149): the
// successive differences along x, y (and z) are exact subtractions on the
// subnormal grid while they stay below 2^23 -- always under the R18 guards
// (|r| < 2^21 in 2D, 2^20 in 3D); the result's bits are sign | |l| and a
// rotate gives v.  Data failing a guard give garbage v (flagged ERANGE).
template <int D>
__device__ __forceinline__ uint32_t lorenzo_md_scaled(float rs, int lane) {
  constexpr int kBX = (D == 3) ? 4 : 8;
  const float px = __shfl_up_sync(kFull, rs, 1);
  float l = (lane % kBX) ? __fsub_rn(rs, px) : rs;            // along x
  const float uy = __shfl_up_sync(kFull, l, kBX);
  if ((lane / kBX) % 4) l = __fsub_rn(l, uy);                 // along y
  if constexpr (D == 3) {
    const float uz = __shfl_up_sync(kFull, l, 16);
    if (lane >= 16) l = __fsub_rn(l, uz);                     // along z
  }
  const uint32_t b = __float_as_uint(l);
  return __funnelshift_l(b, b, 1);
}

// O = Lorenzo order: 1 (the paper's 1D 1-layer predictor) or 2 (2-layer,
// SURVEY 8(f) rank 4; L = 32 only).
// D = Lorenzo dimensions (DESIGN R18): 1 = the paper's 1D
// predictor over consecutive elements; 2 / 3 = blocks of 1x4x8 / 2x4x4 points
// of an (nz, ny, nx) field, gathered into tile order by the producer warp.
// SL = 8 / 16: the byte-granular block lengths (place_small; M = 1): the
// look-back, rings and copy-out count BYTES instead of words.
template <int M, int O, int D = 1, int SL = 0>
__global__ void __launch_bounds__(kCThreads, CUSZP_C_MINBLOCKS) compress_kernel(CompressArgs a) {
  static_assert(O == 1 || (O == 2 && M == 1), "2-layer Lorenzo with L = 32");
  static_assert(D == 1 || (M == 1 && O == 1), "multi-dimensional Lorenzo with L = 32, order 1");
  static_assert(M == 1 || M == 2 || M == 4, "L in {32, 64, 128}");
  static_assert(SL == 0 || ((SL == 8 || SL == 16) && M == 1 && O == 1 && D == 1), "L = 8 / 16");
  constexpr bool kSmall = SL != 0;
  constexpr int kWB = kSmall ? kTileElems / SL / 4 : kTileBlocks / 4;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  CompressSmem<kWB>& sm = *reinterpret_cast<CompressSmem<kWB>*>(smem_raw);
  const int lane = threadIdx.x & 31;
  const int warp = __shfl_sync(0xffffffffu, int(threadIdx.x >> 5), 0);   // provably warp-uniform (no divergence checks before warp-sync ops)
#ifdef CUSZP_TRACE
  // kernel-level points after the per-tile area: [0] first CTA entry, [1] first
  // CTA past pdl_wait, [2] last CTA done (finish), [3] first CTA past the prologue
  uint64_t* tr_k = a.trace ? a.trace + 8ull * a.num_tiles : nullptr;
  if (tr_k && threadIdx.x == 0) atomicMin(reinterpret_cast<unsigned long long*>(tr_k), global_ns());
#endif
  pdl_wait();                                     // range kernel / previous call complete
#ifdef CUSZP_TRACE
  if (tr_k && threadIdx.x == 0) atomicMin(reinterpret_cast<unsigned long long*>(tr_k + 1), global_ns());
#endif
  pdl_launch_dependents();
  const uint32_t epoch = running_epoch(a.ws);

  // ---- eb_abs (Eq 1): ABS -> delta; REL -> lambda * (max - min) over the (min,max) pairs
  float eb = a.eb_in;
  if (a.mode == CUSZP_REL && a.n_pairs == 0) {
    eb = 0.0f;                                      // REL with n = 0 and no range (R11)
  } else if (a.mode == CUSZP_REL) {
    float mn = a.minmax[0], mx = a.minmax[1];
    bool nan = isnan(mn) || isnan(mx);
    for (int p = 1; p < a.n_pairs; ++p) {
      const float lo = a.minmax[2 * p], hi = a.minmax[2 * p + 1];
      nan |= isnan(lo) || isnan(hi);
      if (lo < mn) mn = lo;
      if (hi > mx) mx = hi;
    }
    eb = __fmul_rn(a.eb_in, __fsub_rn(mx, mn));   // R3
    if (nan) eb = __int_as_float(0x7fc00000);
  }
  const float two_eb = __fadd_rn(eb, eb);
  const bool eb_ok = (eb >= kFltMin) && isfinite(two_eb) && a.n > 0;   // R5
  const float recip = __fdiv_rn(1.0f, two_eb);
  float vmax = 0.0f;        // max over this thread's elements of |r0| (R5 guard)
  uint32_t wmax = 0;        // max words of any block (> 25 only for NaN/Inf data)
  const uint64_t p0 = kHdr + align16(a.nb);
  uint32_t* payload = reinterpret_cast<uint32_t*>(a.out + p0);

  if (threadIdx.x == 0) {
    // D > 1: the 32 producer lanes' cp.async groups complete the stage
    for (int s = 0; s < kStages; ++s) { mbar_init(&sm.full[s], D == 1 ? 1 : 32); mbar_init(&sm.empty[s], kCW); }
    for (int m = 0; m < kMeta; ++m) { mbar_init(&sm.staged[m], 1); sm.meta_done[m] = 0; }
    for (int k = 0; k < kTix; ++k) mbar_init(&sm.tixbar[k], 1);
    for (int w = 0; w < kCW; ++w) sm.tail[w] = 0;
    sm.released = 0;
    fence_mbar_init();
  }
  __syncthreads();
#ifdef CUSZP_TRACE
  if (tr_k && threadIdx.x == 0) atomicMin(reinterpret_cast<unsigned long long*>(tr_k + 3), global_ns());
#endif

  if (eb_ok) {
    if (D > 1 && warp == 0) {
      // -------------------------------------------- producer, multi-dim blocks
      // Tile t = blocks 128t .. 128t+127 of the block grid (raster order, x
      // fastest).  Every lane gathers rows of 4 floats of those blocks into
      // the stage in BLOCK order (element j of block i at 32 i + j) with
      // cp.async, zero-filling points outside the field (R8); each lane's
      // copies then complete one of the stage's 32 arrivals.
      constexpr int kBX = (D == 3) ? 4 : 8;
      const bool al16 = (a.nx % 4 == 0) && ((reinterpret_cast<uintptr_t>(a.in) & 15u) == 0);
      for (uint32_t i = 0;; ++i) {
        const int s = int(i % kStages);
        mbar_wait(&sm.empty[s], ((i / kStages) & 1u) ^ 1u);
        uint32_t t = 0;
        if (lane == 0) {
          stress_delay(i);
          t = atomicAdd(&a.ws->ticket, 1u);
        }
        t = __shfl_sync(kFull, t, 0);
        if (t >= a.num_tiles) {
          if (lane == 0) {
            sm.in_tile[s] = kSentinel;  // sync: mbarrier full[s]
            for (uint32_t k = 0; k < uint32_t(kWriters); ++k) {
              sm.tix[(i + k) % kTix] = kSentinel;  // sync: mbarrier tixbar
              mbar_arrive(&sm.tixbar[(i + k) % kTix]);
            }
          }
          __syncwarp();
          mbar_arrive(&sm.full[s]);
          break;
        }
        if (lane == 0) {
          sm.tix[i % kTix] = t;  // sync: mbarrier tixbar
          mbar_arrive(&sm.tixbar[i % kTix]);
          sm.in_tile[s] = t;  // sync: mbarrier full[s]
        }
        const uint32_t dst0 = smem_u32(sm.in[s]);
        // lane l gathers blocks l, l+32, l+64, l+96 of the tile (neighbouring
        // lanes read neighbouring row segments); block coordinates by
        // multiply-shift division (FastDiv; nb < 2^32, checked on the host),
        // row r of the block at a compile-time (z, y, x) step from its origin
        const uint64_t plane = a.ny * a.nx;
#pragma unroll 1
        for (uint32_t ib = lane; ib < uint32_t(kTileBlocks); ib += 32) {
          const uint32_t b = t * uint32_t(kTileBlocks) + ib;
          const uint32_t nbx = uint32_t(a.nbx), nby = uint32_t(a.nby);
          const uint32_t kyz = a.fd_nbx.div(b), kx = b - kyz * nbx;
          const uint32_t kz = a.fd_nby.div(kyz), ky = kyz - kz * nby;
          const bool blk_in = uint64_t(b) < a.nb;
          const uint64_t z0 = uint64_t(kz) * (D == 3 ? 2 : 1), y0 = uint64_t(ky) * 4;
          const uint64_t x0 = uint64_t(kx) * (D == 3 ? 4 : 8);
          const float* org = a.in + (blk_in ? z0 * plane + y0 * a.nx + x0 : 0);
          const uint32_t dst_b = dst0 + 4u * (ib * 32u);
#pragma unroll
          for (uint32_t r = 0; r < 8; ++r) {                          // the block's 8 row segments of 4 points
            // 2D: row r/2, x half r%2 (element (r/2)*8 + 4(r%2)); 3D: z r/4, y r%4 (element 4r)
            const uint32_t rz = (D == 3) ? (r >> 2) : 0u, ry = (D == 3) ? (r & 3u) : (r >> 1);
            const uint32_t rx = (D == 3) ? 0u : 4u * (r & 1u);
            const uint32_t d = (D == 3) ? r * 4 : (r >> 1) * 8 + 4 * (r & 1u);
            const bool row_in = blk_in && z0 + rz < a.nz && y0 + ry < a.ny;
            const float* src = org + (rz ? plane : 0) + ry * a.nx + rx;
            const uint32_t dst = dst_b + 4u * d;
            if (al16) {
              const uint32_t bytes = (row_in && x0 + rx < a.nx) ? 16u : 0u;   // nx % 4 == 0: a row of 4 is all in or all out
              asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(bytes ? src : a.in),
                           "r"(bytes)
                           : "memory");
            } else {
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                const uint32_t bytes = (row_in && x0 + rx + e < a.nx) ? 4u : 0u;
                asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(dst + 4 * e),
                             "l"(bytes ? src + e : a.in), "r"(bytes)
                             : "memory");
              }
            }
          }
        }
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(&sm.full[s])) : "memory");
      }
      (void)kBX;
    } else if (warp == 0) {
      // ------------------------------------------------------------ producer
      if (lane == 0) {
        for (uint32_t i = 0;; ++i) {
          const int s = int(i % kStages);
          mbar_wait(&sm.empty[s], ((i / kStages) & 1u) ^ 1u);
          // ticket taken only once the stage is free: a prefetched ticket would
          // wait a whole tile of compute before its load, and every later tile's
          // look-back would wait for it
          stress_delay(i);
          const uint32_t t = atomicAdd(&a.ws->ticket, 1u);
          if (t >= a.num_tiles) {
            sm.in_tile[s] = kSentinel;  // sync: mbarrier full[s] (arrive release / try_wait acquire)
            mbar_arrive(&sm.full[s]);
            // every writer must see a sentinel: one in each of the next kWriters ticket slots
            for (uint32_t k = 0; k < uint32_t(kWriters); ++k) {
              sm.tix[(i + k) % kTix] = kSentinel;  // sync: mbarrier tixbar
              mbar_arrive(&sm.tixbar[(i + k) % kTix]);
            }
            break;
          }
          sm.tix[i % kTix] = t;                          // writers start the look-back now  // sync: mbarrier tixbar
          mbar_arrive(&sm.tixbar[i % kTix]);
          trace_put(a.trace, t, 0, global_ns());
          sm.in_tile[s] = t;  // sync: mbarrier full[s]
          const uint64_t e0 = uint64_t(t) * kTileElems;
          const uint64_t ne = min(uint64_t(kTileElems), a.n - e0);
          const uint32_t bytes = uint32_t(ne * 4);
          const uint32_t tma_bytes = bytes & ~15u;
          for (uint32_t k = tma_bytes / 4; k < ne; ++k) sm.in[s][k] = a.in[e0 + k];   // <= 3 tail floats  // sync: mbarrier full[s] (the producer's arrive.expect_tx releases them)
          mbar_arrive_expect_tx(&sm.full[s], tma_bytes);
          if (tma_bytes) tma_load_1d(sm.in[s], a.in + e0, tma_bytes, &sm.full[s]);
#if CUSZP_C_L2_AHEAD > 0
          {
            // a third input stage in L2: tickets advance about one grid per
            // round, so the tile CUSZP_C_L2_AHEAD grids ahead is taken (by
            // some CTA) that much later and its TMA then hits L2
            const uint64_t tp = uint64_t(t) + uint64_t(CUSZP_C_L2_AHEAD) * gridDim.x;
            if (tp * kTileElems + kTileElems <= a.n)
              asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a.in + tp * kTileElems), "r"(uint32_t(kTileElems * 4))
                           : "memory");
          }
#endif
        }
      }

    } else if (warp < kFirstCompute) {
      // --------------------------------------- writers (CTA-local tiles j = k, k+W, ...)
      for (uint32_t j = uint32_t(warp - 1);; j += kWriters) {
        const int m = int(j % kMeta);
        const uint32_t par = (j / kMeta) & 1u;
        // the tile's ticket is known as soon as its load is issued: resolve its
        // exclusive prefix (the look-back needs only the predecessors' words)
        // while the tile is still loading and being encoded
        mbar_wait(&sm.tixbar[j % kTix], (j / kTix) & 1u);
        const uint32_t t = sm.tix[j % kTix];  // sync: mbarrier tixbar
        if (t == kSentinel) break;
        uint32_t nw = 0, ns = 0;
#if CUSZP_C_LB_DELAY > 0
        // the tile itself needs a load and an encode (> 4 us) before its
        // prefix matters: do not poll predecessors that early
        __nanosleep(CUSZP_C_LB_DELAY);
#endif
#ifdef CUSZP_TRACE
        const uint64_t t_lb = a.trace ? global_ns() : 0;
#endif
        const uint64_t excl = resolve_excl(a.status, t, epoch, &nw, &ns);
        mbar_wait(&sm.staged[m], par);                      // suspending wait: no issue slots taken
        const TileMeta<kWB>& md = sm.meta[m];
        const uint32_t agg = md.agg;  // sync: mbarrier staged[m]
        if (lane == 0 && t > 0) publish_prefix(a.status, t, excl + agg, epoch);
        auto fbytes = [](uint32_t wb) { return wb - (((wb + 0x7f7f7f7fu) >> 7) & 0x01010101u); };
        if constexpr (kSmall) {
          // F bytes: 512 / 256 per tile, 16 / 8 per lane (plane counts -> F bytewise)
          constexpr uint32_t kPer = uint32_t(kWB) / 32u;
          const uint64_t blk = uint64_t(t) * (kTileElems / SL) + 4u * kPer * lane;
          if (blk < align16(a.nb)) {
            if constexpr (kPer == 4) {
              const uint4 q = *reinterpret_cast<const uint4*>(&md.wb[4 * lane]);  // sync: mbarrier staged[m] after the compute warps' acq_rel count
              *reinterpret_cast<uint4*>(a.out + kHdr + blk) = make_uint4(fbytes(q.x), fbytes(q.y), fbytes(q.z), fbytes(q.w));
            } else {
              const uint2 q = *reinterpret_cast<const uint2*>(&md.wb[2 * lane]);  // sync: mbarrier staged[m] after the compute warps' acq_rel count
              *reinterpret_cast<uint2*>(a.out + kHdr + blk) = make_uint2(fbytes(q.x), fbytes(q.y));
            }
          }
        } else {
          // F bytes of the tile (Fig 12 part 1): lane L converts group L's word
          // counts, F = words - 1 (0 for a zero block) bytewise (counts <= 32, no
          // carries); the stores also cover the F area's zero padding up to
          // align16(nb) (sub-blocks past n encode as zero blocks, F = 0)
          const uint32_t wb = md.wb[lane];  // sync: mbarrier staged[m] after the compute warps' acq_rel count
          const uint32_t f = fbytes(wb);
          const uint64_t blk = (uint64_t(t) * kTileBlocks + 4u * lane) / M;
          if (blk < align16(a.nb)) {
            if constexpr (M == 1) *reinterpret_cast<uint32_t*>(a.out + kHdr + blk) = f;
            else if constexpr (M == 2) *reinterpret_cast<uint16_t*>(a.out + kHdr + blk) = uint16_t(__byte_perm(f, 0, 0x4420u));
            else a.out[kHdr + blk] = uint8_t(f);
          }
        }
        const uint32_t cnt = lane < kCW ? md.cnt[lane] : 0u;  // sync: mbarrier staged[m]
        const uint32_t hd = lane < kCW ? md.head[lane] : 0u;  // sync: mbarrier staged[m]
        uint32_t incl = cnt;
#pragma unroll
        for (int o = 1; o < kCW; o <<= 1) {
          const uint32_t y = __shfl_up_sync(kFull, incl, o);
          if (lane >= o) incl += y;
        }
#ifdef CUSZP_TRACE
        if (lane == 0 && a.trace) {
          trace_put(a.trace, t, 3, t_lb);
          trace_put(a.trace, t, 4, global_ns());
          trace_put(a.trace, t, 5, nw);
          trace_put(a.trace, t, 6, ns);
        }
#endif
        // a8 store: each compute warp's ring segment -> [excl + warp offset, ...):
        // the segment is at most two linear pieces of the ring (before and
        // after its wrap point), each copied with running pointers
        if constexpr (kSmall) {
          // byte segments: the (<= 3) bytes before the first 4-byte aligned
          // destination word and after the last go bytewise (they share words
          // with the neighbouring segments / tiles); the words in between are
          // funnel-shifted out of two ring words
          constexpr uint32_t kMaskB = kRing * 4 - 1;
          const uint8_t* ringb_all = reinterpret_cast<const uint8_t*>(sm.ring);
#pragma unroll 1
          for (int w = 0; w < kCW; ++w) {
            const uint32_t c = __shfl_sync(kFull, cnt, w);
            const uint32_t h = __shfl_sync(kFull, hd, w);
            const uint32_t off = __shfl_sync(kFull, incl - cnt, w);
            const uint8_t* rb = ringb_all + w * (kRing * 4);
            const uint32_t* rw = sm.ring[w];
            uint8_t* g = a.out + p0 + excl + off;
            const uint32_t hb = min(c, uint32_t(-reinterpret_cast<uintptr_t>(g)) & 3u);
            const uint32_t nw = (c - hb) >> 2, tb = c - hb - 4 * nw;
            if (uint32_t(lane) < hb) g[lane] = rb[(h + lane) & kMaskB];  // sync: ring written before staged[m]; reused only after the tail release
            if (uint32_t(lane) < tb) g[hb + 4 * nw + lane] = rb[(h + hb + 4 * nw + lane) & kMaskB];  // sync: ring written before staged[m]; reused only after the tail release
            const uint32_t s0 = h + hb, sh = 8 * (s0 & 3u);
            uint32_t* gw = reinterpret_cast<uint32_t*>(g + hb);
            const uint32_t wm = (s0 >> 2) & (kRing - 1);
            if (wm + nw + 1 <= kRing) {
              // no ring wrap (the common case): unrolled groups of 4 chunks of
              // 32 words with immediate offsets (as the L >= 32 copy-out)
              const uint32_t* src = rw + wm + lane;
              uint32_t* dst = gw + lane;
#pragma unroll
              for (int i = 0; i < 32; i += 4) {
                if (32u * i >= nw) break;
#pragma unroll
                for (int j = i; j < i + 4; ++j)
                  if (lane + 32u * j < nw) dst[32 * j] = __funnelshift_r(src[32 * j], src[32 * j + 1], sh);  // sync: ring written before staged[m]; reused only after the tail release
              }
            } else {
#pragma unroll 2
              for (uint32_t k = lane; k < nw; k += 32) {
                const uint32_t wi = (s0 >> 2) + k;
                const uint32_t lo = rw[wi & (kRing - 1)];  // sync: ring written before staged[m]; reused only after the tail release
                const uint32_t hi = rw[(wi + 1) & (kRing - 1)];  // sync: ring written before staged[m] (bytes past the segment unused)
                gw[k] = __funnelshift_r(lo, hi, sh);
              }
            }
          }
        } else {
        uint32_t* dst_t = payload + excl + lane;
#pragma unroll 1
#ifdef CUSZP_DIAG_NOCOPY
        for (int w = 0; w < 0; ++w) {   // diagnostics only: no copy-out (garbage payload)
#else
        for (int w = 0; w < kCW; ++w) {
#endif
          const uint32_t c = __shfl_sync(kFull, cnt, w);
          const uint32_t h = __shfl_sync(kFull, hd, w);
          const uint32_t off = __shfl_sync(kFull, incl - cnt, w);
          const uint32_t first = min(c, kRing - h);               // words before the wrap
#if CUSZP_C_COPY_UNROLLED
          // a segment is <= 16 x 32 words: groups of 4 chunks, fully unrolled
          // (immediate offsets, a lane test per chunk, one warp-uniform exit
          // test per group; no pointer updates, no remainder loop)
          {
            uint32_t* dst = dst_t + off;
            const uint32_t* src = sm.ring[w] + h + lane;
#pragma unroll
            for (int i = 0; i < kCBPW; i += 4) {
              if (32u * i >= first) break;
#pragma unroll
              for (int j = i; j < i + 4; ++j)
                if (lane + 32u * j < first) dst[32 * j] = src[32 * j];  // sync: ring written before staged[m]; reused only after the tail release
            }
            dst = dst_t + off + first;
            src = sm.ring[w] + lane;
            const uint32_t rest = c - first;
#pragma unroll
            for (int i = 0; i < kCBPW; i += 4) {
              if (32u * i >= rest) break;
#pragma unroll
              for (int j = i; j < i + 4; ++j)
                if (lane + 32u * j < rest) dst[32 * j] = src[32 * j];  // sync: as above
            }
          }
#else
          uint32_t* dst = dst_t + off;
          const uint32_t* src = sm.ring[w] + h + lane;
#pragma unroll 4
          for (int k = lane; k < int(first); k += 32, src += 32, dst += 32) *dst = *src;  // sync: ring written before staged[m]; reused only after the tail release
          src = sm.ring[w] + lane;
          dst = dst_t + off + first;
#pragma unroll 2
          for (int k = lane; k < int(c - first); k += 32, src += 32, dst += 32) *dst = *src;  // sync: ring written before staged[m]; reused only after the tail release
#endif
        }
        }
        // release ring space in CTA tile order
        if (lane == 0) stress_delay(j ^ 0x55u);
        __syncwarp();
        while (ld_volatile_u32(&sm.released) != j) __nanosleep(64);
        if (lane < kCW) sm.tail[lane] += cnt;  // sync: released in tile order after the copy (fence + volatile flag)
        __syncwarp();
        if (lane == 0) {
          __threadfence_block();
          *reinterpret_cast<volatile uint32_t*>(&sm.released) = j + 1;  // sync: fence + volatile flag, polled by the compute warps
        }
        __syncwarp();
      }
    } else {
      // ------------------------------------------------------------ compute
      const int w = warp - kFirstCompute;
      const Xpose xpose(lane);
      // scaled-float Lorenzo (quantize_scaled2) for the paper's default L = 32, order 1
      constexpr bool kScaled = (M == 1 && O == 1);       // L = 32, order 1, any dimensions
      const float kf = lane ? -1.0f : -0.0f;
      const uint64_t nk = (uint64_t(__float_as_uint(kf)) << 32) | __float_as_uint(kf);
      uint32_t head = 0;                                // words this warp has appended (monotonic)
      uint32_t* ring = sm.ring[w];
      for (uint32_t i = 0;; ++i) {
        const int s = int(i % kStages);
        const int m = int(i % kMeta);
#if CUSZP_C_FULL_POLL_NS > 0
        // test + sleep: try_wait's suspension wakes on unrelated barrier
        // traffic (~40 re-tries per wait measured), each re-try costing issue slots
        if (!mbar_test(&sm.full[s], (i / kStages) & 1u)) {
          uint32_t ns = CUSZP_C_FULL_POLL_NS;
          do {
            __nanosleep(ns);
            ns = min(2 * ns, 1024u);
          } while (!mbar_test(&sm.full[s], (i / kStages) & 1u));
        }
#else
        mbar_wait(&sm.full[s], (i / kStages) & 1u);         // suspending wait: no issue slots taken
#endif
        const uint32_t t = sm.in_tile[s];  // sync: mbarrier full[s]
#ifdef CUSZP_TRACE
        // (diagnostics build only: a lane-0 branch here makes ptxas treat the
        // whole encode as possibly divergent -- a divergence check before every
        // warp-synchronous op and 60 % more code)
        if (t != kSentinel && w == 0 && lane == 0) trace_put(a.trace, t, 7, global_ns());
#endif
        // meta slot m free (tile i - kMeta released)
        while (int(i - ld_volatile_u32(&sm.released)) >= kMeta) __nanosleep(CUSZP_C_POLL_NS);
#ifdef CUSZP_TRACE
        if (t != kSentinel && w == 0 && lane == 0) trace_put(a.trace, t, 1, global_ns());
#endif
        if (t == kSentinel) break;                    // the writers stop on the ticket ring
        const uint64_t g0 = uint64_t(t) * kTileElems + uint64_t(w) * kCBPW * 32;   // first element of the warp
        float* src = &sm.in[s][w * kCBPW * 32];
        auto zero_tail = [](float* p, uint64_t g, uint64_t n, int l) { zero_tail_impl<kCBPW * 32>(p, g, n, l); };
        if (D == 1 && t == a.num_tiles - 1) {
          // virtual zero pad (R8): the ragged part of the last tile is zeroed in
          // shared memory once, so the encode loop needs no per-element test.
          // (No TMA writes this stage again in this launch: the producer's next
          // ticket is a sentinel; the proxy fence orders it anyway.)
          zero_tail(src, g0, a.n, lane);                 // out of line: once per launch
        }
        uint32_t cursor = 0;
        // free words in this warp's ring (refreshed only when a worst-case
        // group would not fit)
        uint32_t room = (kSmall ? kRing * 4 : kRing) - (head - ld_volatile_u32(&sm.tail[w]));
        uint32_t wbs[kCBPW / 4];                       // word counts of each group (bytes), for the F array
        if constexpr (kSmall) {
          // L = 8 / 16, one block per lane (kBPL passes of 32 blocks per tile):
          //   a2-a4  R2 quantisation and the block Lorenzo in registers, v = 2|l| + s
          //          (the scaled-subnormal form of quantize_scaled2, in-thread);
          //   a5/a6  planes = bit length of the OR of v (= F + 1; 0: zero block),
          //          c = planes * L/8 bytes (Eq 2), offsets by a warp scan;
          //   a8     the byte sequence 8 planes at a time (gather + 8x8 bit
          //          transpose) funnel-shifted onto 4-byte aligned ring words:
          //          words inside the block are stored, the (<= 2) words shared
          //          with neighbouring blocks are OR-ed into the zeroed ring.
          // each lane encodes the 16 consecutive floats 16 l .. 16 l + 15 of the
          // warp's 512-element slice: kBL = 2 blocks at L = 8, 1 at L = 16
          constexpr int kBL = 16 / SL;
          constexpr int kW = SL / 4;                   // sequence words per 8 planes
          constexpr uint32_t kRB = kRing * 4;          // ring bytes
          uint8_t* fcnt = reinterpret_cast<uint8_t*>(sm.meta[m].wb) + w * (kCBPW * 32 / SL);
          float x[16];
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const float4 f = reinterpret_cast<const float4*>(src + 16 * lane)[q];  // sync: mbarrier full[s] (TMA / producer stores); stage reused after empty[s]
            x[4 * q] = f.x; x[4 * q + 1] = f.y; x[4 * q + 2] = f.z; x[4 * q + 3] = f.w;
          }
          uint32_t v[16];
          float resmax = 0.0f;
          float sc_prev = 0.0f;                        // r_{-1} = 0 (scaled) at each block start
#pragma unroll
          for (int q = 0; q < 8; ++q) {
            if ((2 * q) % SL == 0) sc_prev = 0.0f;
            const uint64_t rs = quantize_scaled2(x[2 * q], x[2 * q + 1], two_eb, recip, vmax, resmax);
            float s0, s1;
            asm("mov.b64 {%0, %1}, %2;" : "=f"(s0), "=f"(s1) : "l"(rs));
            // l = r_j - r_{j-1}, exact on the subnormal grid: bits sign | |l|
            const uint32_t l0 = __float_as_uint(__fsub_rn(s0, sc_prev));
            const uint32_t l1 = __float_as_uint(__fsub_rn(s1, s0));
            v[2 * q] = __funnelshift_l(l0, l0, 1);
            v[2 * q + 1] = __funnelshift_l(l1, l1, 1);
            sc_prev = s1;
          }
          if (__any_sync(kFull, resmax > eb)) {        // R2's correction somewhere in the warp: redo exactly
            uint32_t prev = kRoundMagicBits;
#pragma unroll
            for (int j = 0; j < 16; ++j) {
              if (j % SL == 0) prev = kRoundMagicBits;
              const uint32_t r = quantize_exact(x[j], eb, two_eb, recip, vmax);
              const int l = int(r - prev);
              prev = r;
              v[j] = (uint32_t(l < 0 ? -l : l) << 1) | (uint32_t(l) >> 31);
            }
          }
          uint32_t planes[kBL], c[kBL], ct = 0, pmax = 0;
#pragma unroll
          for (int bb = 0; bb < kBL; ++bb) {
            uint32_t o = 0;
#pragma unroll
            for (int j = 0; j < SL; ++j) o |= v[bb * SL + j];
            planes[bb] = bitlen(o);
            c[bb] = planes[bb] * uint32_t(SL / 8);
            ct += c[bb];
            pmax = max(pmax, planes[bb]);
          }
          if constexpr (kBL == 2) *reinterpret_cast<uint16_t*>(fcnt + 2 * lane) = uint16_t(planes[0] | (planes[1] << 8));  // sync: acq_rel count, then mbarrier staged[m]
          else fcnt[lane] = uint8_t(planes[0]);        // sync: acq_rel count, then mbarrier staged[m]
          wmax = max(wmax, pmax);
          uint32_t incl = ct;
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(kFull, incl, d);
            if (lane >= d) incl += y;
          }
          const uint32_t total = __shfl_sync(kFull, incl, 31);
          while (cursor + total + 4 > room) {          // the tile's bytes (+ the shared word) must fit
            room = kRB - (head - ld_volatile_u32(&sm.tail[w]));
            if (cursor + total + 4 > room) __nanosleep(CUSZP_C_POLL_NS);
          }
          // zero the ring words ahead of the OR-ed shared words (all but a
          // first word shared with the previous tile, whose later bytes are
          // zero already)
          {
            const uint32_t B = head + cursor, E = B + total;
            for (uint32_t k = ((B + 3) >> 2) + lane; k < ((E + 3) >> 2); k += 32) ring[k & (kRing - 1)] = 0u;  // sync: free ring space (room checked); own warp's words
            __syncwarp();
          }
          const uint32_t G = (__reduce_max_sync(kFull, pmax) + 7) >> 3;
          uint32_t X = head + cursor + incl - ct;      // ring byte of the lane's first block
          cursor += total;
#pragma unroll
          for (int bb = 0; bb < kBL; ++bb) {
            const uint32_t sh = 8 * (X & 3u), w0 = X >> 2;
            const uint32_t nwords = c[bb] ? ((X & 3u) + c[bb] + 3) >> 2 : 0u;
            X += c[bb];
            // word j of the block (aligned ring word w0 + j): words 1 .. nwords-2
            // lie inside the block and are stored; word 0 and word nwords-1 may
            // share bytes with the neighbouring blocks and are OR-ed in at the end
            uint32_t first = 0, last = 0;
            auto emit = [&](uint32_t j, uint32_t word) {
              if (j + 1 < nwords) ring[(w0 + j) & (kRing - 1)] = word;  // sync: ring slot freed by the writer's tail release (zeroed); read after staged[m]
              last = (j + 1 == nwords) ? word : last;
            };
            uint32_t prev = 0;
#pragma unroll
            for (int g = 0; g < 4; ++g) {
              if (uint32_t(g) < G) {
                uint32_t sq[kW];
                block_seq8<SL>(v + bb * SL, uint32_t(g), sq);
#pragma unroll
                for (int i = 0; i < kW; ++i) {
                  const uint32_t word = __funnelshift_l(prev, sq[i], sh);
                  if (g == 0 && i == 0) {
                    first = word;
                    last = nwords == 1 ? word : 0u;
                  } else {
                    emit(uint32_t(g * kW + i), word);
                  }
                  prev = sq[i];
                }
              }
            }
            if (G) emit(G * kW, __funnelshift_l(prev, 0u, sh));
            if (nwords) atomicOr(ring + (w0 & (kRing - 1)), first);  // sync: shared with the previous block(s): atomic OR into the zeroed ring
            if (nwords > 1) atomicOr(ring + ((w0 + nwords - 1) & (kRing - 1)), last);  // sync: shared with the next block(s): atomic OR into the zeroed ring
          }
        }
        // Groups of 4 blocks.  The bit transpose packs as many blocks as fit
        // in 32 bits: 4 blocks when every v < 2^8 (F <= 7), 2 when v < 2^16,
        // else 1.  After it, lane q*W + k holds word k of block q (W = 32 /
        // blocks per transpose), and a ballot of the non-zero words gives every
        // block's word count (the top plane is non-zero by definition of F).
#pragma unroll kGUnroll
#ifdef CUSZP_DIAG_NOWORK
        for (int g = 0; g < 0; ++g) {   // diagnostics only: pipeline without the encode work
#else
        for (int g = 0; g < (kSmall ? 0 : kCBPW / 4); ++g) {   // (L = 8 / 16: the per-lane path above)
#endif
          float x[4];
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            x[q] = src[(4 * g + q) * 32 + lane];  // sync: mbarrier full[s] (TMA / cp.async / producer stores); stage reused after empty[s]
          }
          uint32_t r[4];
          float resmax = 0.0f;
          uint64_t rs01 = 0, rs23 = 0;
          if constexpr (kScaled) {
            rs01 = quantize_scaled2(x[0], x[1], two_eb, recip, vmax, resmax);
            rs23 = quantize_scaled2(x[2], x[3], two_eb, recip, vmax, resmax);
          } else {
            quantize_fast2(x[0], x[1], two_eb, recip, vmax, resmax, r[0], r[1]);
            quantize_fast2(x[2], x[3], two_eb, recip, vmax, resmax, r[2], r[3]);
          }
          // NaN residuals are not caught here (fmax drops NaN) but NaN/Inf data
          // always yield a block with > 25 words below (flagged, R5)
#ifdef CUSZP_C_EAGER_RARE
          if (__any_sync(kFull, resmax > eb)) {
#pragma unroll
            for (int q = 0; q < 4; ++q) r[q] = quantize_exact(x[q], eb, two_eb, recip, vmax);
          }
#else
          // the vote is taken now but acted on after the word counts: the
          // Lorenzo shuffles and reductions of the (nearly always exact) fast
          // result do not wait for it; a group that needs R2's correction is
          // then redone in full
          const bool rare = __any_sync(kFull, resmax > eb);
#endif
          uint32_t v[4], wq[4];
          auto counts = [&]() {
            // a5: words per block = bit length of the block's OR of v (= of its max)
#pragma unroll
            for (int q = 0; q < 4; ++q) wq[q] = bitlen(__reduce_or_sync(kFull, v[q]));
          };
          auto lorenzo_and_counts = [&]() {
            if constexpr (M == 1) {
#pragma unroll
              for (int q = 0; q < 4; ++q)
                v[q] = (D > 1) ? lorenzo_md_pack<D>(r[q], lane) : (O == 2) ? lorenzo2_pack(r[q], lane) : lorenzo_pack(r[q], lane);
            } else {
              // a block continues across its sub-blocks: lane 0 of sub-block q
              // takes lane 31 of sub-block q-1 unless q starts a block
#pragma unroll
              for (int q = 0; q < 4; ++q)
                v[q] = lorenzo_pack_first(r[q], lane,
                                          (q % M == 0) ? kRoundMagicBits : __shfl_sync(kFull, r[q > 0 ? q - 1 : 0], 31));
            }
#ifdef CUSZP_DIAG_TINY
            v[0] = v[1] = v[2] = v[3] = 0;   // diagnostics only: all zero blocks (wrong output)
#endif
            counts();
          };
          if constexpr (kScaled) {
            if constexpr (D == 1) {
              lorenzo_scaled2(rs01, nk, v[0], v[1]);
              lorenzo_scaled2(rs23, nk, v[2], v[3]);
            } else {
              float f[4];
              asm("mov.b64 {%0, %1}, %2;" : "=f"(f[0]), "=f"(f[1]) : "l"(rs01));
              asm("mov.b64 {%0, %1}, %2;" : "=f"(f[2]), "=f"(f[3]) : "l"(rs23));
#pragma unroll
              for (int q = 0; q < 4; ++q) v[q] = lorenzo_md_scaled<D>(f[q], lane);
            }
            counts();
          } else {
            lorenzo_and_counts();
          }
#if !defined(CUSZP_C_EAGER_RARE) && !defined(CUSZP_DIAG_NORARE)
          if (rare) {
            if constexpr (kScaled && CUSZP_C_RARE_CALL) {
              const RareOut ro = rare_group_redo<D>(x[0], x[1], x[2], x[3], eb, two_eb, recip, vmax, lane);
              v[0] = ro.v0; v[1] = ro.v1; v[2] = ro.v2; v[3] = ro.v3;
#pragma unroll
              for (int q = 0; q < 4; ++q) wq[q] = (ro.wb >> (8 * q)) & 0xffu;
              vmax = ro.vmax;
            } else {
#pragma unroll
              for (int q = 0; q < 4; ++q) r[q] = quantize_exact(x[q], eb, two_eb, recip, vmax);
              lorenzo_and_counts();
            }
          }
#endif
          // room in this warp's ring for a worst-case group (4 x 32 words)
          while (cursor + 4 * 32 > room) {
            room = kRing - (head - ld_volatile_u32(&sm.tail[w]));
            if (cursor + 4 * 32 > room) __nanosleep(CUSZP_C_POLL_NS);
          }
          if constexpr (M == 2) {                                        // one F per block
            wq[0] = wq[1] = max(wq[0], wq[1]);
            wq[2] = wq[3] = max(wq[2], wq[3]);
          } else if constexpr (M == 4) {
            wq[0] = wq[1] = wq[2] = wq[3] = max(max(wq[0], wq[1]), max(wq[2], wq[3]));
          }
          // > 25 words only for data failing the R5 guard (NaN/Inf, |r0| >= 2^23):
          // flagged ERANGE at the end.  Such garbage blocks still take at most
          // 32 words (v is 32-bit), which the capacity bound covers (DESIGN 9.5).
          const uint32_t span = max(max(wq[0], wq[1]), max(wq[2], wq[3]));
          wmax = max(wmax, span);
          const uint32_t wb = pack4(wq[0], wq[1], wq[2], wq[3]);
          const uint32_t base = head + cursor;
#ifndef CUSZP_DIAG_NOXPOSE   // (diagnostics only: no transposes / ring stores, garbage output)
          if (M > 1) {
            // word k of sub-block q -> block payload position M k + q % M
            const uint32_t pb = wb * 0x01010100u;                       // exclusive byte prefix (sums <= 100)
            if (span <= 8) {
              const uint32_t tw = xpose(pack4(v[0], v[1], v[2], v[3]));
              const uint32_t q = uint32_t(lane) >> 3, k = lane & 7;
              const uint32_t pre = __byte_perm(pb, 0, 0x4440u + (q & ~uint32_t(M - 1)));
              if (k < __byte_perm(wb, 0, 0x4440u + q)) ring[(base + pre + M * k + (q & (M - 1))) & (kRing - 1)] = tw;  // sync: ring slot freed by the writer's tail release; read after staged[m]
            } else if (span <= 16) {
              const uint32_t t01 = xpose(__byte_perm(v[0], v[1], 0x5410u));
              const uint32_t t23 = xpose(__byte_perm(v[2], v[3], 0x5410u));
              const uint32_t h = lane >= 16 ? 1u : 0u, k = lane & 15;
              if (k < wq[0]) ring[(base + M * k + h) & (kRing - 1)] = t01;  // sync: ring slot freed by the writer's tail release; read after staged[m]
              const uint32_t pre23 = (M == 2) ? wq[0] + wq[1] : 0u;
              const uint32_t sub23 = (M == 2) ? h : 2u + h;
              if (k < wq[2]) ring[(base + pre23 + M * k + sub23) & (kRing - 1)] = t23;  // sync: ring slot freed by the writer's tail release; read after staged[m]
            } else {
#pragma unroll
              for (int q = 0; q < 4; ++q) {
                const uint32_t tq = xpose(v[q]);
                const uint32_t pre = (q & ~(M - 1)) == 0 ? 0u : __byte_perm(pb, 0, 0x4440u + (q & ~(M - 1)));
                if (uint32_t(lane) < wq[q]) ring[(base + pre + M * uint32_t(lane) + (q & (M - 1))) & (kRing - 1)] = tq;  // sync: ring slot freed by the writer's tail release; read after staged[m]
              }
            }
          } else if (span <= 8) {
            const uint32_t tw = xpose(pack4(v[0], v[1], v[2], v[3]));
            const uint32_t pb = wb * 0x01010100u;                       // exclusive byte prefix (sums <= 24)
            const uint32_t sel = 0x4440u + (uint32_t(lane) >> 3), k = lane & 7;
            if (k < __byte_perm(wb, 0, sel)) ring[(base + __byte_perm(pb, 0, sel) + k) & (kRing - 1)] = tw;  // sync: ring slot freed by the writer's tail release; read after staged[m]
#ifdef CUSZP_DIAG_NOSPAN32
          } else {   // diagnostics only: no 1-block-per-transpose path (wrong output when a span > 16)
#else
          } else if (span <= 16) {
#endif
            const uint32_t t01 = xpose(__byte_perm(v[0], v[1], 0x5410u));
            const uint32_t t23 = xpose(__byte_perm(v[2], v[3], 0x5410u));
            const bool hi = lane >= 16;
            const uint32_t k = lane & 15;
            if (k < (hi ? wq[1] : wq[0])) ring[(base + (hi ? wq[0] : 0u) + k) & (kRing - 1)] = t01;  // sync: ring slot freed by the writer's tail release; read after staged[m]
            if (k < (hi ? wq[3] : wq[2])) ring[(base + wq[0] + wq[1] + (hi ? wq[2] : 0u) + k) & (kRing - 1)] = t23;  // sync: ring slot freed by the writer's tail release; read after staged[m]
#ifdef CUSZP_DIAG_NOSPAN32
          }
          if (false) {
#endif
          } else if constexpr (CUSZP_C_RARE_CALL && kScaled) {
            store_singles(ring, base, v[0], v[1], v[2], v[3], wb, lane);   // span > 16: rare, out of line
          } else {
            uint32_t o = base;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const uint32_t tq = xpose(v[q]);
              if (uint32_t(lane) < wq[q]) ring[(o + lane) & (kRing - 1)] = tq;  // sync: ring slot freed by the writer's tail release; read after staged[m]
              o += wq[q];
            }
          }
#endif
          cursor += (wb * 0x01010101u) >> 24;                          // sum of the 4 counts
#if CUSZP_C_GUNROLL >= 4
          wbs[g] = wb;
#else
          if (lane == 0) sm.meta[m].wb[w * (kCBPW / 4) + g] = wb;  // sync: acq_rel count, then mbarrier staged[m]
#endif
        }
        __syncwarp();
        if (elect_one()) {                                 // lane 0 (elect: no warp-aggregated atomic below)
          mbar_arrive(&sm.empty[s]);                       // input stage consumed
          TileMeta<kWB>& md = sm.meta[m];
          // the group word counts go to the writer, which stores the tile's F bytes
#if CUSZP_C_GUNROLL >= 4
          if constexpr (kSmall) {}                       // F bytes stored per block (small path)
          else if constexpr (kCBPW / 4 == 4) *reinterpret_cast<uint4*>(&md.wb[w * 4]) = make_uint4(wbs[0], wbs[1], wbs[2], wbs[3]);  // sync: acq_rel count, then mbarrier staged[m]; slot reused after released
          else *reinterpret_cast<uint2*>(&md.wb[w * 2]) = make_uint2(wbs[0], wbs[1]);  // sync: acq_rel count, then mbarrier staged[m]
#endif
          md.cnt[w] = uint16_t(cursor);  // sync: acq_rel count, then mbarrier staged[m]; slot reused after released
          md.head[w] = uint16_t(head & ((kSmall ? 4 * kRing : kRing) - 1));  // sync: acq_rel count, then mbarrier staged[m]; slot reused after released
          uint32_t done;                                   // release: cnt/head before the count; acquire: the others'
          asm volatile("atom.acq_rel.cta.shared::cta.add.u32 %0, [%1], 1;"
                       : "=r"(done) : "r"(smem_u32(&sm.meta_done[m])) : "memory");
          if (done == kCW - 1) {
            // last warp of the tile: aggregate -> publish at once (look-back, part 1)
            uint32_t agg = 0;
#pragma unroll
            for (int k = 0; k < kCW; ++k)
              agg += *reinterpret_cast<volatile uint16_t*>(&md.cnt[k]);  // sync: atom.acq_rel on meta_done[m] (the last warp acquires every warp's count)
            publish_aggregate(a.status, t, agg, epoch);
            trace_put(a.trace, t, 2, global_ns());
            md.tile = t;  // sync: the last warp, then mbarrier staged[m]
            md.agg = agg;  // sync: the last warp, then mbarrier staged[m]; slot reused after released
            sm.meta_done[m] = 0;
            mbar_arrive(&sm.staged[m]);
          }
        }
        head += cursor;
      }
    }
  }

  // R5 guard: some |r0| >= 2^22 (NaN and Inf included)
  uint32_t flag = 0;
  if (!eb_ok) flag = (a.n > 0) ? kBadRange : 0u;
  else if (!(vmax < (O == 2 || D == 2 ? 0.5f * kGuard : D == 3 ? 0.25f * kGuard : kGuard)) ||
           wmax > uint32_t(kMaxBlockWords))
    flag = kBadRange;   // R5 / R17 / R18

  if (cta_finish(a.ws, flag)) {
    uint32_t final_status = CUSZP_OK;
    if (threadIdx.x == 0) {
      const uint32_t acc = *reinterpret_cast<volatile uint32_t*>(&a.ws->status_accum);
      if (acc & kBadRange) final_status = CUSZP_ERANGE;
      uint64_t total_words = 0;
      if (final_status == CUSZP_OK && a.num_tiles > 0)
        total_words = ld_relaxed_u64(a.status + a.num_tiles - 1) & kValueMask;
      const uint64_t payload_bytes = final_status == CUSZP_OK ? total_words * (kSmall ? 1 : 4) : 0;   // L = 8 / 16 count bytes
      uint8_t* h = a.out;                                   // header (R10)
      *reinterpret_cast<uint32_t*>(h) = 0x505A5343u;        // "CSZP"
      h[4] = CUSZP_VERSION;
      h[5] = uint8_t(a.mode | (O == 2 ? 0x10 : 0) | ((D - 1) << 5));   // predictor order (R17), dims (R18)
      h[6] = uint8_t(final_status);
      h[7] = uint8_t(SL == 8 ? 3 : SL == 16 ? 4 : 5 + (M == 2 ? 1 : M == 4 ? 2 : 0));   // log2(L)
      *reinterpret_cast<uint64_t*>(h + 8) = a.n;
      // R11: n = 0 records the bound that would have been used (a sharded
      // REL shard's global lambda * range; 0 for a lone empty REL array)
      *reinterpret_cast<float*>(h + 16) = a.mode == CUSZP_REL ? eb : a.eb_in;
      *reinterpret_cast<float*>(h + 20) = a.eb_in;
      *reinterpret_cast<uint64_t*>(h + 24) = payload_bytes;
      if (a.out_bytes) *a.out_bytes = (a.n == 0) ? uint64_t(kHdr) : p0 + payload_bytes;
    }
    finish_call(a.ws, a.status, a.status_cap, epoch, final_status);
#ifdef CUSZP_TRACE
    if (tr_k && threadIdx.x == 0) tr_k[2] = global_ns();
#endif
  }
}

namespace {
template <int M, int O = 1, int D = 1, int SL = 0>
cudaError_t configure_m(int* occ) {
  constexpr int kWB = SL ? kTileElems / SL / 4 : kTileBlocks / 4;
  const int smem = int(sizeof(CompressSmem<kWB>));
  cudaError_t e = cudaFuncSetAttribute(compress_kernel<M, O, D, SL>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, compress_kernel<M, O, D, SL>, kCThreads, smem);
  return e;
}
template <int M, int O = 1, int D = 1, int SL = 0>
cudaError_t launch_k(cudaLaunchConfig_t cfg, const CompressArgs& a) {
  constexpr int kWB = SL ? kTileElems / SL / 4 : kTileBlocks / 4;
  cfg.dynamicSmemBytes = sizeof(CompressSmem<kWB>);
  return cudaLaunchKernelEx(&cfg, compress_kernel<M, O, D, SL>, a);
}
}  // namespace

// L in {8, 16, 32, 64, 128}: resident CTAs per SM of that block length's kernel
cudaError_t compress_configure(int L, int* occ) {
  int occ2 = 0;
  if (L == 32 && (configure_m<1, 2>(&occ2) != cudaSuccess || configure_m<1, 1, 2>(&occ2) != cudaSuccess ||
                  configure_m<1, 1, 3>(&occ2) != cudaSuccess))
    return cudaErrorUnknown;
  switch (L) {
    case 8: return configure_m<1, 1, 1, 8>(occ);
    case 16: return configure_m<1, 1, 1, 16>(occ);
    case 32: return configure_m<1>(occ);
    case 64: return configure_m<2>(occ);
    default: return configure_m<4>(occ);
  }
}

cudaError_t compress_launch(int L, int order, unsigned grid, const CompressArgs& a, cudaStream_t s) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kCThreads);
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;   // see pdl_wait()
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  if (a.dims == 2) return launch_k<1, 1, 2>(cfg, a);
  if (a.dims == 3) return launch_k<1, 1, 3>(cfg, a);
  if (order == 2) return launch_k<1, 2>(cfg, a);
  switch (L) {
    case 8: return launch_k<1, 1, 1, 8>(cfg, a);
    case 16: return launch_k<1, 1, 1, 16>(cfg, a);
    case 32: return launch_k<1, 1>(cfg, a);
    case 64: return launch_k<2, 1>(cfg, a);
    default: return launch_k<4, 1>(cfg, a);
  }
}

size_t compress_smem_bytes() { return sizeof(CompressSmem<kTileBlocks / 4>); }
int compress_threads() { return kCThreads; }

}  // namespace cuszp
