// internal.cuh -- device-side definitions shared by the three kernels of the
// B200-native cuSZp path (sm_100a).  Nothing here is shared with oracle/.
//
// Design: persistent, warp-specialised CTAs take TILES of
// 128 L-blocks (4096 elements, 16 KB of fp32) by atomic ticket.  A producer
// warp streams tiles HBM -> shared memory with 1D TMA bulk copies into an
// mbarrier ring; compute warps own 16 blocks each with one lane per element
// (lane j <-> element j), so the paper's per-block steps become warp
// primitives (Lorenzo = shfl_up, max = redux.max, F = clz, bit-shuffle =
// a 13-instruction warp bit-transpose that handles 1, 2 or 4 blocks at once); a
// scan warp places each tile with a decoupled look-back (the paper's
// chained scan) over epoch-tagged status words, so no memset is
// needed between calls and the look-back latency overlaps the next tile.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/cuszp.h"

namespace cuszp {

constexpr int kL = CUSZP_BLOCK_LEN;           // R1
constexpr int kHdr = CUSZP_HEADER_BYTES;      // R10
constexpr float kGuard = 4194304.0f;          // 2^22 (R5)
constexpr float kRoundMagic = 12582912.0f;    // 1.5 * 2^23
constexpr uint32_t kRoundMagicBits = 0x4B400000u;
constexpr int kMaxF = 24;
constexpr float kFltMin = 1.17549435e-38f;
constexpr uint32_t kFull = 0xffffffffu;

// Tile geometry (both scan kernels).
constexpr int kComputeWarps = 8;
constexpr int kBPW = 16;                                  // L-blocks per compute warp per tile
constexpr int kTileBlocks = kComputeWarps * kBPW;         // 128 blocks = 4096 elements
constexpr int kTileElems = kTileBlocks * 32;
constexpr int kMaxBlockWords = kMaxF + 1;                 // sign map + 24 planes
constexpr uint32_t kSentinel = 0xffffffffu;

// ---------------------------------------------------------------- workspace
struct WsCtrl {
  uint32_t epoch;          // tag of the status words of the last scan kernel
  uint32_t ticket;         // tile ticket counter, 0 between calls
  uint32_t exit_count;     // finished CTAs, 0 between calls
  uint32_t status_accum;   // async status bits of the running call, 0 between calls
  uint32_t last_status;    // cuszp_status of the last finished call
  uint32_t range_max_key;  // atomicMax of order-preserving keys (0 = identity)
  uint32_t range_min_key;  // atomicMax of ~key (0 = identity)
  uint32_t range_exit;     // range kernel exit counter
  float minmax[2];         // result of the last range kernel
  uint32_t pad[22];
};
static_assert(sizeof(WsCtrl) == 128, "ws ctrl layout");
constexpr size_t kWsCtrlBytes = 128;

// async status bits (status_accum)
constexpr uint32_t kBadRange = 1u;     // -> CUSZP_ERANGE
constexpr uint32_t kBadCorrupt = 2u;   // -> CUSZP_ECORRUPT

// Look-back status word: [63:41] epoch | [40] inclusive-prefix flag |
// [39:0] value in 4-byte words.  A word whose epoch differs from the
// running call's is "not yet published".
constexpr int kEpochShift = 41;
constexpr uint64_t kPrefixFlag = 1ull << 40;
constexpr uint64_t kValueMask = (1ull << 40) - 1;
constexpr uint32_t kMaxEpoch = (1u << 23) - 1;

__host__ __device__ inline uint64_t align16(uint64_t v) { return (v + 15u) & ~uint64_t(15); }

// ------------------------------------------------------------ memory helpers
__device__ __forceinline__ void st_relaxed_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ float ld_stream_f32(const float* p) {
  float v;
  asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ float4 ld_stream_f32x4(const float4* p) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "l"(p));
  return v;
}

// ------------------------------------------------------- mbarrier / TMA bulk
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
// Blocks until the phase with the given parity has completed.  try_wait
// suspends the warp in hardware (it stops competing for issue slots) until
// the phase completes or the suspend-time hint (ns) expires.
#ifndef CUSZP_SUSPEND_NS
#define CUSZP_SUSPEND_NS 100000
#endif
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
      " @!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(parity), "n"(CUSZP_SUSPEND_NS)
      : "memory");
}
// One suspending try (true once the phase has completed).
__device__ __forceinline__ bool mbar_try(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n"
      " selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity), "n"(CUSZP_SUSPEND_NS)
      : "memory");
  return ok != 0;
}
// Non-blocking probe: has the phase with the given parity completed?
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n"
      " mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      " selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
// Named (hardware) barriers: waiting warps are descheduled and cost no issue
// slots, unlike polling loops over mbarriers (which every mbarrier event in
// the CTA wakes).  count = all participating threads (multiple of 32).
__device__ __forceinline__ void named_sync(uint32_t id, uint32_t count) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
__device__ __forceinline__ void named_arrive(uint32_t id, uint32_t count) {
  asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(count) : "memory");
}
// 1D TMA bulk copy global -> shared (UBLKCP); 16-byte aligned, size % 16 == 0.
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// ------------------------------------------------------------- bit transpose
// 32x32 bit-matrix transpose across a warp (lane r holds row r; afterwards
// lane k holds the word whose bit j is bit k of the old row j).  Five
// butterfly stages, each ONE shuffle plus a per-lane-constant merge: the
// 16- and 8-bit stages are a single byte permute (PRMT) with a per-lane
// selector, the 4/2/1-bit stages a rotate + 3-input LOP with a per-lane
// rotate amount and keep-mask, so both halves of every exchange execute the
// same instruction (no divergence): 13 instructions per transpose.
// This is the paper's Block Bit-shuffle done for 32 elements
// at once, and -- being an involution up to layout -- also its inverse.
struct Xpose {
  uint32_t sel16, sel8;
  uint32_t amt[3];
  uint32_t keep[3];
  __device__ __forceinline__ explicit Xpose(int lane) {
    // PRMT(x, partner): low half keeps its low bytes and takes the partner's
    // low ones (16: [x0 x1 p0 p1], 8: [x0 p0 x2 p2]); high half mirrors it.
    sel16 = (lane & 16) ? 0x3276u : 0x5410u;
    sel8 = (lane & 8) ? 0x3715u : 0x6240u;
    const uint32_t m[3] = {0x0F0F0F0Fu, 0x33333333u, 0x55555555u};
#pragma unroll
    for (int s = 0; s < 3; ++s) {
      const int j = 4 >> s;
      const bool low = (lane & j) == 0;
      amt[s] = low ? uint32_t(j) : uint32_t(32 - j);
      keep[s] = low ? m[s] : ~m[s];
    }
  }
  __device__ __forceinline__ uint32_t operator()(uint32_t x) const {
    x = __byte_perm(x, __shfl_xor_sync(0xffffffffu, x, 16), sel16);
    x = __byte_perm(x, __shfl_xor_sync(0xffffffffu, x, 8), sel8);
#pragma unroll
    for (int s = 0; s < 3; ++s) {
      const uint32_t t = __shfl_xor_sync(0xffffffffu, x, 4 >> s);
      const uint32_t r = __funnelshift_l(t, t, amt[s]);   // rotate left
      x = (x & keep[s]) | (r & ~keep[s]);
    }
    return x;
  }
};

// --------------------------------------------- programmatic dependent launch
// The scan kernels are launched with programmatic stream serialisation: their
// CTAs may be scheduled while the previous kernel's CTAs retire, and wait here
// (before touching anything that kernel wrote) for its completion and memory.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
// Lets the next (PDL-launched) kernel be scheduled as this grid's CTAs retire.
__device__ __forceinline__ void pdl_launch_dependents() { asm volatile("griddepcontrol.launch_dependents;" :::); }

// ------------------------------------------------------------- diagnostics
__device__ __forceinline__ uint64_t global_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
// trace[8 t + slot] = value (only when a trace buffer was installed)
__device__ __forceinline__ void trace_put(uint64_t* trace, uint32_t t, int slot, uint64_t v) {
  if (trace) trace[8ull * t + slot] = v;
}

// Look-back stress build (-DCUSZP_STRESS, tests/test_gpu_stress.py): a
// pseudo-random delay (1 call in 4, up to ~4 us) before every status-word
// publication, ticket and ring release, so predecessors publish out of order
// and late, exercising every path of the look-back and of the ring
// bookkeeping.  Compiled out of the production library.
#ifdef CUSZP_STRESS
__device__ __forceinline__ void stress_delay(uint32_t salt) {
  uint32_t h = salt * 0x9E3779B1u ^ uint32_t(global_ns()) ^ (blockIdx.x * 0x85EBCA6Bu);
  h ^= h >> 15;
  h *= 0x2C1B3C6Du;
  h ^= h >> 12;
  if ((h & 3u) == 0) __nanosleep(h >> 20);
}
#else
__device__ __forceinline__ void stress_delay(uint32_t) {}
#endif

// ------------------------------------------------------------- warp helpers
// one lane of a converged warp (elect.sync): unlike `lane == 0`, ptxas then
// knows a single lane runs the block and emits its shared-memory atomics
// as they are (no warp-aggregation sequence around them)
__device__ __forceinline__ bool elect_one() {
  uint32_t p;
  asm volatile("{ .reg .pred P; elect.sync _|P, 0xffffffff; selp.u32 %0, 1, 0, P; }" : "=r"(p));
  return p != 0;
}
// sum over the warp of values < 2^44 (look-back parts: <= K aggregates /
// prefixes of <= 40 bits): two 32-bit REDUX.SUMs of the low 24 and the high
// bits (each sum fits 32 bits) instead of five 64-bit shuffle rounds
__device__ __forceinline__ uint64_t warp_sum_u44(uint64_t v) {
  const uint32_t lo = __reduce_add_sync(kFull, uint32_t(v) & 0xFFFFFFu);
  const uint32_t hi = __reduce_add_sync(kFull, uint32_t(v >> 24));
  return (uint64_t(hi) << 24) + lo;
}
__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
  return v;
}

// Epoch used by the running scan kernel (ws->epoch is only written by the
// last CTA of the previous kernel, which completed before this one began).
__device__ __forceinline__ uint32_t running_epoch(const WsCtrl* ws) {
  const uint32_t e = *reinterpret_cast<const volatile uint32_t*>(&ws->epoch);
  return e + 1;   // in [1, kMaxEpoch]; the last CTA resets ws->epoch to 0 at kMaxEpoch
}

// Decoupled look-back (single pass; the paper's "chained-scan
// parallelization", refs [22],[37]), split in two so that the
// aggregate is published the moment it is known and the (latency-bound)
// prefix resolution runs on a warp of its own.
//
// publish_aggregate: one thread; tile 0's aggregate is already its prefix.
__device__ __forceinline__ void publish_aggregate(uint64_t* status, uint32_t t, uint64_t agg,
                                                  uint32_t epoch) {
  const uint64_t tag = uint64_t(epoch) << kEpochShift;
  stress_delay(t * 2u);
  st_relaxed_u64(status + t, tag | (t == 0 ? kPrefixFlag : 0ull) | agg);
}

// resolve_prefix: all 32 lanes of one warp.  Inspects predecessors in
// windows of 32*K (K status words per lane, loads in flight together), stops
// at the nearest inclusive prefix, publishes tile t's inclusive prefix and
// returns its exclusive prefix (in 4-byte words).  Polling backs off
// exponentially: thousands of warps may be waiting at once, and their loads
// share the L2 with the data streams.
#ifndef CUSZP_LB_K
#define CUSZP_LB_K 1
#endif
#ifndef CUSZP_LB_BACKOFF_MIN
#define CUSZP_LB_BACKOFF_MIN 64
#endif
#ifndef CUSZP_LB_BACKOFF_MAX
#define CUSZP_LB_BACKOFF_MAX 1024
#endif
// resolve_excl: the look-back proper (all 32 lanes): tile t's exclusive
// prefix, without publishing anything.  It needs only the predecessors'
// words, so it may run before tile t's own aggregate is known.
__device__ __forceinline__ uint64_t resolve_excl(const uint64_t* status, uint32_t t, uint32_t epoch,
                                                 uint32_t* n_windows = nullptr, uint32_t* n_spins = nullptr) {
  if (t == 0) return 0;
  constexpr int K = CUSZP_LB_K;
  static_assert(K >= 1 && K <= 16, "a lane's part (<= K values of 40 bits) must stay below 2^44 (warp_sum_u44)");
  uint32_t windows = 0, spins = 0;
  const int lane = threadIdx.x & 31;
  const uint64_t tag = uint64_t(epoch) << kEpochShift;
  uint64_t excl = 0;
  int64_t top = int64_t(t) - 1;          // nearest predecessor not yet summed
  uint32_t backoff = CUSZP_LB_BACKOFF_MIN;
  while (true) {
    uint64_t w[K];
    while (true) {
      bool ready = true;
#pragma unroll
      for (int k = 0; k < K; ++k) {
        const int64_t idx = top - K * lane - k;   // distance K*lane + k from `top`
        w[k] = (idx >= 0) ? ld_relaxed_u64(status + idx) : (tag | kPrefixFlag);
        ready &= (w[k] >> kEpochShift) == epoch;
      }
      if (__all_sync(kFull, ready)) break;
      ++spins;
      __nanosleep(backoff);
      backoff = min(backoff * 2u, uint32_t(CUSZP_LB_BACKOFF_MAX));
    }
    ++windows;
    // per lane: aggregates up to and including its first prefix (k = distance order)
    uint64_t part = 0;
    bool has_p = false;
#pragma unroll
    for (int k = 0; k < K; ++k) {
      if (!has_p) {
        part += w[k] & kValueMask;
        has_p = (w[k] & kPrefixFlag) != 0;
      }
    }
    const uint32_t pmask = __ballot_sync(kFull, has_p);
    const int stop = pmask ? (__ffs(pmask) - 1) : 31;
    excl += warp_sum_u44(lane <= stop ? part : 0ull);
    if (pmask) break;
    top -= 32 * K;
  }
  if (n_windows) *n_windows = windows;
  if (n_spins) *n_spins = spins;
  return excl;
}

// publish_prefix: one thread; tile t's inclusive prefix.
__device__ __forceinline__ void publish_prefix(uint64_t* status, uint32_t t, uint64_t incl, uint32_t epoch) {
  stress_delay(t * 2u + 1u);
  st_relaxed_u64(status + t, (uint64_t(epoch) << kEpochShift) | kPrefixFlag | incl);
}

__device__ __forceinline__ uint64_t resolve_prefix(uint64_t* status, uint32_t t, uint64_t agg,
                                                   uint32_t epoch, uint32_t* n_windows = nullptr,
                                                   uint32_t* n_spins = nullptr) {
  if (t == 0) return 0;
  const uint64_t excl = resolve_excl(status, t, epoch, n_windows, n_spins);
  if ((threadIdx.x & 31) == 0) publish_prefix(status, t, excl + agg, epoch);
  return excl;
}

// Inclusive scan step with the hardware's in-range predicate (SHFL + @p IADD,
// no select): x += x[lane - o] when that lane lies in the same segment.
// seg_c = (32 - segment width) << 8.
__device__ __forceinline__ int scan_step_up(int x, int o, int seg_c) {
  asm volatile(
      "{\n .reg .pred p;\n .reg .b32 t;\n"
      " shfl.sync.up.b32 t|p, %0, %1, %2, 0xffffffff;\n"
      " @p add.s32 %0, %0, t;\n}"
      : "+r"(x)
      : "r"(o), "r"(seg_c));
  return x;
}

// The same step on subnormal-scaled floats (decompress, order 1): exact as
// long as every partial sum stays on the subnormal grid.
__device__ __forceinline__ float scan_step_up_f(float x, int o, int seg_c) {
  asm volatile(
      "{\n .reg .pred p;\n .reg .b32 t;\n"
      " shfl.sync.up.b32 t|p, %0, %1, %2, 0xffffffff;\n"
      " @p add.rn.f32 %0, %0, t;\n}"
      : "+f"(x)
      : "r"(o), "r"(seg_c));
  return x;
}

// End-of-kernel bookkeeping: accumulate this CTA's status bits, count the
// CTA out; returns true (in every thread) for the last CTA to finish.
__device__ __forceinline__ bool cta_finish(WsCtrl* ws, uint32_t bad_bits) {
  __shared__ int s_last;
  const uint32_t any = __syncthreads_or(bad_bits);
  if (threadIdx.x == 0) {
    if (any) {
      // collect the distinct bits of the CTA
      atomicOr(&ws->status_accum, any);
    }
    __threadfence();
    const uint32_t prev = atomicAdd(&ws->exit_count, 1u);
    s_last = (prev == gridDim.x - 1);
  }
  __syncthreads();
  const bool last = s_last != 0;
  if (last) __threadfence();
  return last;
}

// Last CTA: reset the per-call counters, advance the epoch; at the epoch
// limit clear every status word so the next epoch (1) can never alias.
__device__ __forceinline__ void finish_call(WsCtrl* ws, uint64_t* status, uint32_t status_cap,
                                            uint32_t epoch, uint32_t final_status) {
  if (epoch >= kMaxEpoch) {
    for (uint32_t i = threadIdx.x; i < status_cap; i += blockDim.x) status[i] = 0;
    __syncthreads();
    epoch = 0;
  }
  if (threadIdx.x == 0) {
    ws->last_status = final_status;
    ws->status_accum = 0;
    ws->ticket = 0;
    ws->exit_count = 0;
    ws->epoch = epoch;
    __threadfence();
  }
}

// ------------------------------------------------------------ kernel params
// Division by a launch-invariant 32-bit divisor d >= 1 (Granlund-Montgomery,
// round-up multiplier): q = (t + ((n - t) >> s1)) >> s2, t = umulhi(n, m),
// exact for every 32-bit n.  The multi-dimensional block coordinates use it
// instead of a ~20-instruction integer division per block.
struct FastDiv {
  uint32_t m = 1, s1 = 0, s2 = 0;
  FastDiv() = default;
  __host__ explicit FastDiv(uint32_t d) {
    uint32_t l = 0;
    while (l < 32 && (uint64_t(1) << l) < d) ++l;                     // ceil(log2 d)
    m = uint32_t(((uint64_t(1) << 32) * ((uint64_t(1) << l) - d)) / d + 1);
    s1 = l < 1 ? l : 1;
    s2 = l > 1 ? l - 1 : 0;
  }
  __device__ __forceinline__ uint32_t div(uint32_t n) const {
    const uint32_t t = __umulhi(n, m);
    return (t + ((n - t) >> s1)) >> s2;
  }
};

struct CompressArgs {
  const float* in;
  uint64_t n;
  uint64_t nb;
  uint32_t num_tiles;
  int mode;                  // 0 ABS, 1 REL
  float eb_in;               // delta (ABS) or lambda (REL)
  const float* minmax;       // REL: n_pairs (min, max) pairs on the device
  int n_pairs;
  uint8_t* out;
  unsigned long long* out_bytes;
  WsCtrl* ws;
  uint64_t* status;
  uint32_t status_cap;
  uint64_t* trace;           // diagnostics only (nullptr): 8 u64 per tile, see tools/trace_scan.py
  int dims;                  // Lorenzo dimensions (R18): 1, or 2 / 3 over the (nz, ny, nx) field below
  uint64_t nz, ny, nx;       // field shape (dims > 1; n = nz ny nx)
  uint64_t nby, nbx;         // block grid rows / columns (dims > 1; nb = nbz nby nbx)
  FastDiv fd_nbx, fd_nby;    // division by nbx / nby (dims > 1)
};

struct DecompressArgs {
  const uint8_t* in;
  uint64_t in_bytes;
  float* out;
  uint64_t n;
  uint64_t nb;
  uint32_t num_tiles;
  WsCtrl* ws;
  uint64_t* status;
  uint32_t status_cap;
  uint64_t* trace;
  int dims;                  // as CompressArgs
  uint64_t nz, ny, nx;
  uint64_t nby, nbx;
  FastDiv fd_nbx, fd_nby;
  uint32_t chunk_tiles;      // tiles per look-back chunk: 8 for large inputs, 4 for small ones (balance)
};

struct RangeArgs {
  const float* in;
  uint64_t n;
  float* user_minmax;
  WsCtrl* ws;
};

struct QualityArgs {
  const float* x;            // original
  const float* y;            // reconstruction
  uint64_t n;
  double bound;              // count |x - y| > bound (negative: counts every point with |x - y| > bound)
  double* out;               // cuszp_quality on the device (14 x 8 bytes)
  void* ws;                  // [0,128) counter, then one 128-byte partial per CTA
};
constexpr int kQualityMaxGrid = 2048;

// Kernels templated on M = L / 32 are launched through these host wrappers
// defined next to them (compress.cu / decompress.cu): M in {1, 2, 4}.
cudaError_t compress_configure(int L, int* occupancy);        // smem attribute + CTAs per SM (L = block length)
cudaError_t compress_launch(int L, int order, unsigned grid, const CompressArgs& a, cudaStream_t s);
cudaError_t decompress_configure(int L, int* occupancy);
cudaError_t decompress_launch(int L, int order, unsigned grid, const DecompressArgs& a, cudaStream_t s);
// L in {8, 16}, diagnostics build only (-DCUSZP_SMALL_L_3PASS, small_l.cu): the
// round-1 three-launch path, the A/B baseline of the one-pass kernels.
cudaError_t compress_small_launch(int L, const CompressArgs& a, cudaStream_t s);
cudaError_t decompress_small_launch(int L, const DecompressArgs& a, cudaStream_t s);
__global__ void quality_kernel(QualityArgs a);
__global__ void range_kernel(RangeArgs a);
int launch_copy_len(void* dst, const void* src, const unsigned long long* d_len, uint64_t cap,
                    unsigned long long* len_out, int sms, cudaStream_t s);
int launch_stream_len(const void* h_stream_dev, uint64_t n, unsigned long long* d_len, cudaStream_t s);
int launch_container_put(const void* shard, const void* hdr, uint32_t P, uint32_t p, void* cont, int write_header,
                         int sms, cudaStream_t s);
size_t compress_smem_bytes();
int compress_threads();
size_t decompress_smem_bytes();
int decompress_threads();

}  // namespace cuszp
