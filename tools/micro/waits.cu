// Microbenchmark (diagnostics): how long do the waiting primitives really
// sleep on sm_100a?  One warp waits on an mbarrier that another warp completes
// after ~20 us of clock spinning; we count wait-loop iterations.
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ bool test(uint64_t* b, uint32_t par) {
  uint32_t ok; asm volatile("{.reg .pred p; mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}" : "=r"(ok) : "r"(sa(b)), "r"(par) : "memory"); return ok;
}
template <int HINT> __device__ __forceinline__ bool trywait(uint64_t* b, uint32_t par) {
  uint32_t ok;
  if (HINT) asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3; selp.u32 %0,1,0,p;}" : "=r"(ok) : "r"(sa(b)), "r"(par), "n"(HINT) : "memory");
  else asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}" : "=r"(ok) : "r"(sa(b)), "r"(par) : "memory");
  return ok;
}
template <int MODE, int NS>
__global__ void k(unsigned long long* out) {
  __shared__ uint64_t bar;
  if (threadIdx.x == 0) { asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(sa(&bar))); asm volatile("fence.mbarrier_init.release.cluster;"); }
  __syncthreads();
  unsigned long long it = 0;
  if (threadIdx.x / 32 == 1) {
    long long t0 = clock64(); while (clock64() - t0 < 40000) {}
    if (threadIdx.x == 32) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(sa(&bar)) : "memory");
  } else if (threadIdx.x / 32 == 0) {
    if (MODE == 0) { while (!test(&bar, 0)) { ++it; if (NS) __nanosleep(NS); } }
    if (MODE == 1) { while (!trywait<0>(&bar, 0)) ++it; }
    if (MODE == 2) { while (!trywait<NS>(&bar, 0)) ++it; }
    if (threadIdx.x == 0) out[0] = it;
  }
}
int main() {
  unsigned long long* d; cudaMalloc(&d, 8); unsigned long long h;
  auto run = [&](auto kern, const char* name) { kern<<<1, 64>>>(d); cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost); printf("%-28s iterations over ~20us: %llu\n", name, h); };
  run(k<0, 0>, "test, no sleep");
  run(k<0, 32>, "test + nanosleep(32)");
  run(k<0, 128>, "test + nanosleep(128)");
  run(k<0, 1000>, "test + nanosleep(1000)");
  run(k<0, 5000>, "test + nanosleep(5000)");
  run(k<1, 0>, "try_wait (no hint)");
  run(k<2, 1000>, "try_wait hint 1000ns");
  run(k<2, 100000>, "try_wait hint 100000ns");
  return 0;
}
