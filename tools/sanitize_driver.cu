// sanitize_driver.cu -- a torch-free driver of the C ABI for compute-sanitizer
// (memcheck / racecheck / synccheck / initcheck) runs of the look-back
// kernels.  Built and run by
// tests/test_gpu_stress.py:
//     nvcc -gencode arch=compute_100a,code=sm_100a -o sanitize_driver \
//          tools/sanitize_driver.cu -Iinclude -Lpaper_conf_sc_huangd0lc23_b200 -lcuszp
//     compute-sanitizer --tool memcheck ./sanitize_driver
//
// Every buffer is allocated with its EXACT size (so any read or write past
// an end is an out-of-bounds access the sanitizer sees); inputs are a smooth
// 1D field (C1's recipe, written out here) at ragged sizes; each round trip
// must satisfy the error bound |x - x'| <= eb + ulp(x).  The
// compressed streams are decompressed from exact-size copies (in_bytes = S).
// Exit code 0 = every check passed.
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include <cuda_runtime.h>

#include "cuszp.h"

#define CK(x)                                                                              \
  do {                                                                                     \
    cudaError_t e_ = (x);                                                                  \
    if (e_ != cudaSuccess) {                                                               \
      std::fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); \
      std::exit(2);                                                                        \
    }                                                                                      \
  } while (0)
#define OKS(x)                                                                             \
  do {                                                                                     \
    int s_ = (x);                                                                          \
    if (s_ != CUSZP_OK) {                                                                  \
      std::fprintf(stderr, "%s:%d %s -> %s\n", __FILE__, __LINE__, #x, cuszp_status_string(s_)); \
      std::exit(3);                                                                        \
    }                                                                                      \
  } while (0)

extern "C" void cuszp_debug_set_grid(int compress_grid, int decompress_grid);

static int round_trip(size_t n, float eb, int mode, int L, int order) {
  std::vector<float> x(n);
  const double tau = 6.283185307179586;
  for (size_t i = 0; i < n; ++i) {
    const double t = double(i) / double(n ? n : 1);
    x[i] = float(std::sin(tau * 3 * t) + 0.5 * std::sin(tau * 11 * t + 1.0) + 0.25 * std::sin(tau * 37 * t + 2.0) +
                 1e-5 * double((i * 2654435761u) % 1000) / 1000.0);
  }
  float *d_x = nullptr, *d_y = nullptr;
  void *d_out = nullptr, *d_ws = nullptr, *d_exact = nullptr;
  unsigned long long* d_len = nullptr;
  const size_t cap = cuszp_max_compressed_bytes_L(n, L), wsb = cuszp_workspace_bytes(n);
  CK(cudaMalloc(&d_x, (n ? n : 1) * sizeof(float)));
  CK(cudaMalloc(&d_y, (n ? n : 1) * sizeof(float)));
  CK(cudaMalloc(&d_out, cap));
  CK(cudaMalloc(&d_ws, wsb));
  CK(cudaMalloc(&d_len, 8));
  CK(cudaMemset(d_ws, 0, wsb));
  CK(cudaMemcpy(d_x, x.data(), n * sizeof(float), cudaMemcpyHostToDevice));
  OKS(cuszp_compress_ex(d_x, n, eb, mode, L, order, d_out, cap, d_len, d_ws, wsb, nullptr));
  unsigned long long S = 0;
  CK(cudaMemcpy(&S, d_len, 8, cudaMemcpyDeviceToHost));
  int st = cuszp_last_status(d_ws, nullptr);
  int bad = 0;
  if (st != CUSZP_OK) {
    std::fprintf(stderr, "n=%zu L=%d order=%d: compress status %s\n", n, L, order, cuszp_status_string(st));
    bad = 1;
    S = 32;
  }
  // decompress from an exact-size copy of the stream (every read must stay inside S bytes)
  CK(cudaMalloc(&d_exact, S));
  CK(cudaMemcpy(d_exact, d_out, S, cudaMemcpyDeviceToDevice));
  std::vector<float> y(n);
  cuszp_header h;
  if (!bad) {
    OKS(cuszp_decompress_ex(d_exact, S, d_y, n, L, order, d_ws, wsb, nullptr));
    st = cuszp_last_status(d_ws, nullptr);
    CK(cudaMemcpy(y.data(), d_y, n * sizeof(float), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&h, d_exact, 32, cudaMemcpyDeviceToHost));
    bad = (st != CUSZP_OK);
  }
  if (!bad && S > 33) {
    // a stream cut by one byte, in an exact-size allocation: ECORRUPT, no read past it
    void* d_cut = nullptr;
    CK(cudaMalloc(&d_cut, S - 1));
    CK(cudaMemcpy(d_cut, d_out, S - 1, cudaMemcpyDeviceToDevice));
    OKS(cuszp_decompress_ex(d_cut, S - 1, d_y, n, L, order, d_ws, wsb, nullptr));
    if (cuszp_last_status(d_ws, nullptr) != CUSZP_ECORRUPT) {
      std::fprintf(stderr, "n=%zu L=%d order=%d: truncated stream not ECORRUPT\n", n, L, order);
      bad = 1;
    }
    CK(cudaFree(d_cut));
    OKS(cuszp_decompress_ex(d_exact, S, d_y, n, L, order, d_ws, wsb, nullptr));   // the full stream again
    CK(cudaMemcpy(y.data(), d_y, n * sizeof(float), cudaMemcpyDeviceToHost));
  }
  for (size_t i = 0; i < n && !bad; ++i) {
    const double ulp = double(std::nextafterf(std::fabs(x[i]), INFINITY)) - std::fabs(double(x[i]));
    if (std::fabs(double(x[i]) - double(y[i])) > double(h.eb_abs) + ulp) {
      std::fprintf(stderr, "n=%zu L=%d order=%d: bound violated at %zu\n", n, L, order, i);
      bad = 1;
    }
  }
  CK(cudaFree(d_x));
  CK(cudaFree(d_y));
  CK(cudaFree(d_out));
  CK(cudaFree(d_ws));
  CK(cudaFree(d_len));
  CK(cudaFree(d_exact));
  return bad;
}

int main(int argc, char** argv) {
  int fails = 0;
  const size_t sizes[] = {1, 31, 33, 4095, 4097, 100003, (size_t(1) << 20) + 11};
  for (size_t n : sizes) {
    if (n > 1) fails += round_trip(n, 1e-4f, CUSZP_REL, 32, 1);     // n = 1 is a constant field: ERANGE by R5
    fails += round_trip(n, 1e-3f, CUSZP_ABS, 32, 1);
  }
  fails += round_trip(100003, 1e-4f, CUSZP_REL, 64, 1);
  fails += round_trip(100003, 1e-4f, CUSZP_REL, 128, 1);
  fails += round_trip(100003, 1e-4f, CUSZP_REL, 32, 2);
  fails += round_trip(100003, 1e-4f, CUSZP_REL, 8, 1);
  fails += round_trip(100003, 1e-4f, CUSZP_REL, 16, 1);
  // persistent grids of 1, 3 and 4 x SMs CTAs (look-back across every kind of residency)
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  for (int g : {1, 3, 4 * sms}) {
    cuszp_debug_set_grid(g, g);
    fails += round_trip(100003, 1e-4f, CUSZP_REL, 32, 1);
    fails += round_trip(100003, 1e-4f, CUSZP_REL, 8, 1);
  }
  cuszp_debug_set_grid(0, 0);
  CK(cudaDeviceSynchronize());
  std::printf("sanitize_driver: %d failure(s)\n", fails);
  return fails ? 1 : 0;
}
