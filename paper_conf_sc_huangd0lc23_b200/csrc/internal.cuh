// internal.cuh -- device-side definitions shared by the three kernels of the
// B200-native cuSZp path (sm_100a).  Nothing here is shared with oracle/.
//
// Design: persistent CTAs take TILES of 64 L-blocks
// (8 warps x 8 blocks) by atomic ticket; within a warp one lane owns one
// element of a 32-element block (lane j <-> element j), so the paper's
// per-block steps become warp primitives: Lorenzo = shfl_up, sign map and
// bit planes = ballot, max = redux.max, F = 32 - clz.  Tiles are placed by
// a decoupled look-back scan (the paper's chained scan) whose
// status words are epoch-tagged so no memset is needed between calls.
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
constexpr int kWarps = 8;                     // warps per CTA
constexpr int kThreads = kWarps * 32;
constexpr int kBPW = 8;                       // L-blocks per warp per tile
constexpr int kTileBlocks = kWarps * kBPW;    // 64 blocks = 2048 elements per tile

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

// ------------------------------------------------------------- warp helpers
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
// parallelization", refs [22],[37]).  Called by all 32 lanes of
// ONE warp of the CTA owning tile t with that tile's aggregate `agg` (in
// 4-byte words).  Publishes the aggregate, walks predecessors 32 at a
// time, publishes the inclusive prefix and returns the exclusive one.
__device__ __forceinline__ uint64_t tile_lookback(uint64_t* status, uint32_t t, uint64_t agg,
                                                  uint32_t epoch) {
  const int lane = threadIdx.x & 31;
  const uint64_t tag = uint64_t(epoch) << kEpochShift;
  if (t == 0) {
    if (lane == 0) st_relaxed_u64(status, tag | kPrefixFlag | agg);
    return 0;
  }
  if (lane == 0) st_relaxed_u64(status + t, tag | agg);
  uint64_t excl = 0;
  int64_t base = int64_t(t) - 1;
  while (true) {
    const int64_t idx = base - lane;
    uint64_t w;
    int spins = 0;
    while (true) {
      w = (idx >= 0) ? ld_relaxed_u64(status + idx) : (tag | kPrefixFlag);
      const bool ready = (w >> kEpochShift) == epoch;
      if (__all_sync(kFull, ready)) break;
      if (++spins > 4) __nanosleep(64);
    }
    const uint32_t pmask = __ballot_sync(kFull, (w & kPrefixFlag) != 0);
    const int stop = pmask ? (__ffs(pmask) - 1) : 31;
    excl += warp_sum_u64(lane <= stop ? (w & kValueMask) : 0);
    if (pmask) break;
    base -= 32;
  }
  if (lane == 0) st_relaxed_u64(status + t, tag | kPrefixFlag | (excl + agg));
  return excl;
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
};

struct RangeArgs {
  const float* in;
  uint64_t n;
  float* user_minmax;
  WsCtrl* ws;
};

__global__ void compress_kernel(CompressArgs a);
__global__ void decompress_kernel(DecompressArgs a);
__global__ void range_kernel(RangeArgs a);

}  // namespace cuszp
