// cuszp_abi.cu -- host side of the C ABI declared in include/cuszp.h:
// argument validation, workspace / buffer sizing, persistent grid sizing,
// kernel launches.  Never allocates, never synchronises (except the three
// documented synchronous helpers), so every async call is graph-capturable.
#include <cstring>
#include <mutex>

#include "internal.cuh"

using namespace cuszp;

namespace {

uint64_t num_blocks(uint64_t n, int L = kL) { return (n + L - 1) / L; }
// M = L / 32 for the block lengths of SURVEY 8(f) rank 3 (0: unsupported)
int sub_blocks(int L) { return L == 32 ? 1 : L == 64 ? 2 : L == 128 ? 4 : 0; }
// index of a block length in the per-L occupancy tables (8, 16, 32, 64, 128)
int lidx(int L) { return L == 8 ? 0 : L == 16 ? 1 : L == 32 ? 2 : L == 64 ? 3 : 4; }
// L = 8 / 16: byte-granular planes, the one-thread-per-block path (small_l.cu)
bool small_L(int L) { return L == 8 || L == 16; }
bool valid_L(int L) { return sub_blocks(L) != 0 || small_L(L); }
uint64_t num_tiles(uint64_t n) { return (num_blocks(n) + kTileBlocks - 1) / kTileBlocks; }

struct DeviceInfo {
  int sms = 0;
  int occ_compress = 0, occ_decompress = 0, occ_range = 0, occ_quality = 0;
  int occ_c[5] = {0, 0, 0, 0, 0};   // compress, per L = 8, 16, 32, 64, 128
  int occ_d[5] = {0, 0, 0, 0, 0};   // decompress, per L = 8, 16, 32, 64, 128
};

// Per-device launch geometry, computed once: persistent grids of
// (SM count x resident CTAs per SM) for the two scan kernels.
int device_info(DeviceInfo* out) {
  static std::mutex mu;
  static DeviceInfo cache[64];
  static bool have[64] = {false};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return CUSZP_ECUDA;
  std::lock_guard<std::mutex> lock(mu);
  if (!have[dev]) {
    DeviceInfo d;
    if (cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return CUSZP_ECUDA;
    for (int k = 0; k < 5; ++k)
      if (compress_configure(8 << k, &d.occ_c[k]) != cudaSuccess) return CUSZP_ECUDA;
    for (int k = 0; k < 5; ++k)
      if (decompress_configure(8 << k, &d.occ_d[k]) != cudaSuccess) return CUSZP_ECUDA;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&d.occ_range, range_kernel, 256, 0) != cudaSuccess ||
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&d.occ_quality, quality_kernel, 256, 0) != cudaSuccess)
      return CUSZP_ECUDA;
    d.occ_compress = d.occ_c[2];
    d.occ_decompress = d.occ_d[2];
    cache[dev] = d;
    have[dev] = true;
  }
  *out = cache[dev];
  return CUSZP_OK;
}

bool misaligned(const void* p, uintptr_t a) { return (reinterpret_cast<uintptr_t>(p) & (a - 1)) != 0; }

bool eb_is_normal(float eb) {
  if (!(eb >= kFltMin)) return false;
  const float two = eb + eb;
  return two - two == 0.0f;   // finite
}

// Diagnostics: a device buffer of 8 u64 per tile filled by the next launches
// (tools/trace_scan.py).  Not part of include/cuszp.h; nullptr in production.
uint64_t* g_trace = nullptr;
// Diagnostics: persistent grid sizes forced by cuszp_debug_set_grid (0 = the
// occupancy-derived default); used by the look-back stress tests.
int g_grid_compress = 0, g_grid_decompress = 0;

// Decompression look-back chunk: 8 tiles once every CTA of the persistent
// grid gets >= 24 tiles (the scanner's per-chunk latency then hides behind
// the decode; measured -13 % on the 1.1 GB field), else 4 (balance on small
// inputs: 8-tile chunks cost +5..15 % at 100 MB).  DESIGN sec 8.1.
uint32_t decompress_chunk_tiles(uint64_t tiles, uint64_t grid) { return tiles >= 24 * grid ? 8u : 4u; }

uint32_t status_capacity(size_t ws_bytes) {
  const uint64_t c = (ws_bytes - kWsCtrlBytes) / 8;
  return c > 0xffffffffull ? 0xffffffffu : uint32_t(c);
}

// Multi-dimensional Lorenzo (R18): block box and block grid of a field.
struct MdGrid {
  int dims = 1;
  uint64_t nz = 1, ny = 1, nx = 0, nbz = 0, nby = 0, nbx = 0, nb = 0;
};
bool md_grid(size_t nz, size_t ny, size_t nx, int dims, MdGrid* g) {
  if ((dims != 2 && dims != 3) || nz == 0 || ny == 0 || nx == 0) return false;
  g->dims = dims;
  g->nz = nz; g->ny = ny; g->nx = nx;
  const uint64_t bz = dims == 3 ? 2 : 1, bx = dims == 3 ? 4 : 8;
  g->nbz = (nz + bz - 1) / bz;
  g->nby = (ny + 3) / 4;
  g->nbx = (nx + bx - 1) / bx;
  g->nb = g->nbz * g->nby * g->nbx;
  return g->nb < (uint64_t(1) << 32) && nz * ny * nx / nz / ny == nx;   // 32-bit block ids; no overflow
}

int launch_compress(const float* d_in, size_t n, int mode, float eb_in, const float* d_minmax,
                    int n_pairs, void* d_out, size_t out_capacity, unsigned long long* d_out_bytes,
                    void* d_ws, size_t ws_bytes, cudaStream_t stream, int L = kL, int order = 1,
                    const MdGrid* md = nullptr) {
  const int M = sub_blocks(L);
  if (!valid_L(L) || (order != 1 && order != 2) || (order == 2 && M != 1)) return CUSZP_EINVAL;
  const uint64_t nb = md ? md->nb : num_blocks(n, L);
  // tiles of 128 blocks of 32 elements (4096 elements; M sub-blocks per L-block)
  const uint64_t tiles = md ? (nb + kTileBlocks - 1) / kTileBlocks : num_tiles(n);
  if (out_capacity < (md ? size_t(kHdr + align16(nb) + 128 * nb) : cuszp_max_compressed_bytes_L(n, L)) ||
      ws_bytes < kWsCtrlBytes + 8 * (tiles > 0 ? tiles : 1))
    return CUSZP_ENOSPACE;
  DeviceInfo di;
  if (device_info(&di) != CUSZP_OK) return CUSZP_ECUDA;
  CompressArgs a;
  a.in = d_in;
  a.n = n;
  a.nb = nb;
  a.num_tiles = uint32_t(tiles);
  a.dims = md ? md->dims : 1;
  a.nz = md ? md->nz : 1;
  a.ny = md ? md->ny : 1;
  a.nx = md ? md->nx : n;
  a.nby = md ? md->nby : 1;
  a.nbx = md ? md->nbx : nb;
  if (md) {
    a.fd_nbx = FastDiv(uint32_t(md->nbx));
    a.fd_nby = FastDiv(uint32_t(md->nby));
  }
  a.mode = mode;
  a.eb_in = eb_in;
  a.minmax = d_minmax;
  a.n_pairs = n_pairs;
  a.out = static_cast<uint8_t*>(d_out);
  a.out_bytes = d_out_bytes;
  a.ws = static_cast<WsCtrl*>(d_ws);
  a.status = reinterpret_cast<uint64_t*>(static_cast<uint8_t*>(d_ws) + kWsCtrlBytes);
  a.status_cap = status_capacity(ws_bytes);
  a.trace = g_trace;
#ifdef CUSZP_SMALL_L_3PASS
  // diagnostics build: the three-launch L = 8 / 16 path (small_l.cu), for A/B
  if (small_L(L)) return compress_small_launch(L, a, stream) == cudaSuccess ? CUSZP_OK : CUSZP_ECUDA;
#endif
  const int occ = di.occ_c[lidx(L)];
  uint64_t grid = uint64_t(di.sms) * uint64_t(occ > 0 ? occ : 1);
  if (g_grid_compress > 0) grid = uint64_t(g_grid_compress);
  if (grid > a.num_tiles) grid = a.num_tiles;
  if (grid < 1) grid = 1;
  return compress_launch(L, order, unsigned(grid), a, stream) == cudaSuccess ? CUSZP_OK : CUSZP_ECUDA;
}

}  // namespace

extern "C" {

size_t cuszp_max_compressed_bytes(size_t n) { return cuszp_max_compressed_bytes_L(n, kL); }

size_t cuszp_max_compressed_bytes_L(size_t n, int block_len) {
  if (!valid_L(block_len)) return 0;
  // a valid block takes at most 25 words (F <= 24, R5); a block of data that
  // fails the guard is only known to be ERANGE at the end of the kernel and
  // may take 32 (v is 32-bit): the bound covers that too (DESIGN 9.5)
  const uint64_t nb = num_blocks(n, block_len);
  return size_t(kHdr + align16(nb) + uint64_t(block_len / 8) * 32u * nb);
}

size_t cuszp_compressed_bytes_from_F(const uint8_t* h_F, size_t nb) {
  uint64_t s = kHdr + align16(nb);
  for (size_t k = 0; k < nb; ++k)
    if (h_F[k]) s += 4u * (uint64_t(h_F[k]) + 1u);
  return size_t(s);
}

size_t cuszp_workspace_bytes(size_t n) {
  const uint64_t t = num_tiles(n);
  return size_t(kWsCtrlBytes + 8 * (t > 0 ? t : 1));
}

int cuszp_range(const float* d_in, size_t n, float* d_minmax, void* d_ws, size_t ws_bytes, void* stream) {
  if (d_in == nullptr || d_ws == nullptr || n == 0 || (reinterpret_cast<uintptr_t>(d_in) & 3u))
    return CUSZP_EINVAL;
  if (ws_bytes < kWsCtrlBytes) return CUSZP_ENOSPACE;
  DeviceInfo di;
  if (device_info(&di) != CUSZP_OK) return CUSZP_ECUDA;
  RangeArgs a{d_in, n, d_minmax, static_cast<WsCtrl*>(d_ws)};
  const uint64_t want = (n / 4 + 255) / 256;   // one float4 per thread at most
  uint64_t grid = uint64_t(di.sms) * uint64_t(di.occ_range > 0 ? di.occ_range : 1);
  if (grid > want) grid = want;
  if (grid < 1) grid = 1;
  range_kernel<<<unsigned(grid), 256, 0, static_cast<cudaStream_t>(stream)>>>(a);
  return cudaGetLastError() == cudaSuccess ? CUSZP_OK : CUSZP_ECUDA;
}

size_t cuszp_quality_workspace_bytes(void) { return 128 + 128 * size_t(kQualityMaxGrid); }

int cuszp_quality(const float* d_x, const float* d_y, size_t n, double bound, cuszp_quality_stats* d_q, void* d_ws,
                  size_t ws_bytes, void* stream) {
  static_assert(sizeof(cuszp_quality_stats) == 14 * 8, "cuszp_quality_stats layout");
  if (d_x == nullptr || d_y == nullptr || d_q == nullptr || d_ws == nullptr || n == 0 ||
      ((reinterpret_cast<uintptr_t>(d_x) | reinterpret_cast<uintptr_t>(d_y)) & 3u) ||
      (reinterpret_cast<uintptr_t>(d_q) & 7u) || (reinterpret_cast<uintptr_t>(d_ws) & 15u) || bound != bound)
    return CUSZP_EINVAL;
  if (ws_bytes < cuszp_quality_workspace_bytes()) return CUSZP_ENOSPACE;
  DeviceInfo di;
  if (device_info(&di) != CUSZP_OK) return CUSZP_ECUDA;
  QualityArgs a{d_x, d_y, n, bound, reinterpret_cast<double*>(d_q), d_ws};
  const uint64_t want = (n / 8 + 255) / 256;   // two float4 pairs per thread at most
  uint64_t grid = uint64_t(di.sms) * uint64_t(di.occ_quality > 0 ? di.occ_quality : 1);
  if (grid > want) grid = want;
  if (grid > uint64_t(kQualityMaxGrid)) grid = kQualityMaxGrid;
  if (grid < 1) grid = 1;
  quality_kernel<<<unsigned(grid), 256, 0, static_cast<cudaStream_t>(stream)>>>(a);
  return cudaGetLastError() == cudaSuccess ? CUSZP_OK : CUSZP_ECUDA;
}

int cuszp_compress(const float* d_in, size_t n, float eb, int mode, void* d_out, size_t out_capacity,
                   unsigned long long* d_out_bytes, void* d_ws, size_t ws_bytes, void* stream) {
  return cuszp_compress_L(d_in, n, eb, mode, kL, d_out, out_capacity, d_out_bytes, d_ws, ws_bytes, stream);
}

int cuszp_compress_L(const float* d_in, size_t n, float eb, int mode, int block_len, void* d_out,
                     size_t out_capacity, unsigned long long* d_out_bytes, void* d_ws, size_t ws_bytes,
                     void* stream) {
  return cuszp_compress_ex(d_in, n, eb, mode, block_len, 1, d_out, out_capacity, d_out_bytes, d_ws, ws_bytes,
                           stream);
}

int cuszp_compress_ex(const float* d_in, size_t n, float eb, int mode, int block_len, int order, void* d_out,
                      size_t out_capacity, unsigned long long* d_out_bytes, void* d_ws, size_t ws_bytes,
                      void* stream) {
  if ((n > 0 && d_in == nullptr) || d_out == nullptr || d_ws == nullptr || !valid_L(block_len) ||
      (order != 1 && order != 2) || (order == 2 && block_len != kL))
    return CUSZP_EINVAL;
  if ((reinterpret_cast<uintptr_t>(d_in) & 15u) || (reinterpret_cast<uintptr_t>(d_out) & 15u) ||
      (reinterpret_cast<uintptr_t>(d_ws) & 15u))
    return CUSZP_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (mode == CUSZP_ABS) {
    if (!eb_is_normal(eb)) return CUSZP_EINVAL;
    return launch_compress(d_in, n, CUSZP_ABS, eb, nullptr, 0, d_out, out_capacity, d_out_bytes, d_ws,
                           ws_bytes, s, block_len, order);
  }
  if (mode == CUSZP_REL) {
    if (!(eb > 0.0f) || !(eb - eb == 0.0f)) return CUSZP_EINVAL;
    if (out_capacity < cuszp_max_compressed_bytes_L(n, block_len) || ws_bytes < cuszp_workspace_bytes(n))
      return CUSZP_ENOSPACE;
    const WsCtrl* ws = static_cast<const WsCtrl*>(d_ws);
    if (n > 0) {
      const int st = cuszp_range(d_in, n, nullptr, d_ws, ws_bytes, stream);
      if (st != CUSZP_OK) return st;
    }
    return launch_compress(d_in, n, CUSZP_REL, eb, n > 0 ? ws->minmax : nullptr, n > 0 ? 1 : 0, d_out,
                           out_capacity, d_out_bytes, d_ws, ws_bytes, s, block_len, order);
  }
  return CUSZP_EINVAL;
}

int cuszp_compress_minmax(const float* d_in, size_t n, float lambda, const float* d_minmax, int n_pairs,
                          void* d_out, size_t out_capacity, unsigned long long* d_out_bytes, void* d_ws,
                          size_t ws_bytes, void* stream) {
  return cuszp_compress_minmax_L(d_in, n, lambda, d_minmax, n_pairs, kL, d_out, out_capacity, d_out_bytes, d_ws,
                                 ws_bytes, stream);
}

int cuszp_compress_minmax_L(const float* d_in, size_t n, float lambda, const float* d_minmax, int n_pairs,
                            int block_len, void* d_out, size_t out_capacity, unsigned long long* d_out_bytes,
                            void* d_ws, size_t ws_bytes, void* stream) {
  if ((n > 0 && d_in == nullptr) || d_out == nullptr || d_ws == nullptr || d_minmax == nullptr ||
      n_pairs <= 0 || !valid_L(block_len))
    return CUSZP_EINVAL;
  if ((reinterpret_cast<uintptr_t>(d_in) & 15u) || (reinterpret_cast<uintptr_t>(d_out) & 15u) ||
      (reinterpret_cast<uintptr_t>(d_ws) & 15u))
    return CUSZP_EINVAL;
  if (!(lambda > 0.0f) || !(lambda - lambda == 0.0f)) return CUSZP_EINVAL;
  return launch_compress(d_in, n, CUSZP_REL, lambda, d_minmax, n_pairs, d_out, out_capacity, d_out_bytes,
                         d_ws, ws_bytes, static_cast<cudaStream_t>(stream), block_len);
}

int cuszp_decompress(const void* d_in, size_t in_bytes, float* d_out, size_t n, void* d_ws, size_t ws_bytes,
                     void* stream) {
  return cuszp_decompress_L(d_in, in_bytes, d_out, n, kL, d_ws, ws_bytes, stream);
}

int cuszp_decompress_L(const void* d_in, size_t in_bytes, float* d_out, size_t n, int block_len, void* d_ws,
                       size_t ws_bytes, void* stream) {
  return cuszp_decompress_ex(d_in, in_bytes, d_out, n, block_len, 1, d_ws, ws_bytes, stream);
}

int cuszp_decompress_ex(const void* d_in, size_t in_bytes, float* d_out, size_t n, int block_len, int order,
                        void* d_ws, size_t ws_bytes, void* stream) {
  const int M = sub_blocks(block_len);
  if (d_in == nullptr || (n > 0 && d_out == nullptr) || d_ws == nullptr || !valid_L(block_len) ||
      (order != 1 && order != 2) || (order == 2 && M != 1))
    return CUSZP_EINVAL;
  if ((reinterpret_cast<uintptr_t>(d_in) & 15u) || (reinterpret_cast<uintptr_t>(d_out) & 15u) ||
      (reinterpret_cast<uintptr_t>(d_ws) & 15u))
    return CUSZP_EINVAL;
  if (ws_bytes < cuszp_workspace_bytes(n)) return CUSZP_ENOSPACE;
  DeviceInfo di;
  if (device_info(&di) != CUSZP_OK) return CUSZP_ECUDA;
  DecompressArgs a;
  a.in = static_cast<const uint8_t*>(d_in);
  a.in_bytes = in_bytes;
  a.out = d_out;
  a.n = n;
  a.nb = num_blocks(n, block_len);
  a.num_tiles = uint32_t(num_tiles(n));
  a.ws = static_cast<WsCtrl*>(d_ws);
  a.status = reinterpret_cast<uint64_t*>(static_cast<uint8_t*>(d_ws) + kWsCtrlBytes);
  a.status_cap = status_capacity(ws_bytes);
  a.trace = g_trace;
  a.dims = 1;
  a.nz = a.ny = 1;
  a.nx = n;
  a.nby = 1;
  a.nbx = a.nb;
#ifdef CUSZP_SMALL_L_3PASS
  // diagnostics build: the three-launch L = 8 / 16 path (small_l.cu), for A/B
  if (small_L(block_len))
    return decompress_small_launch(block_len, a, static_cast<cudaStream_t>(stream)) == cudaSuccess ? CUSZP_OK
                                                                                                : CUSZP_ECUDA;
#endif
  const int occ = di.occ_d[lidx(block_len)];
  uint64_t grid = uint64_t(di.sms) * uint64_t(occ > 0 ? occ : 1);
  if (g_grid_decompress > 0) grid = uint64_t(g_grid_decompress);
  a.chunk_tiles = decompress_chunk_tiles(a.num_tiles, grid);
  if (grid > a.num_tiles) grid = a.num_tiles;
  if (grid < 1) grid = 1;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  return decompress_launch(block_len, order, unsigned(grid), a, s) == cudaSuccess ? CUSZP_OK : CUSZP_ECUDA;
}

size_t cuszp_num_blocks_md(size_t nz, size_t ny, size_t nx, int dims) {
  MdGrid g;
  return md_grid(nz, ny, nx, dims, &g) ? size_t(g.nb) : 0;
}

size_t cuszp_max_compressed_bytes_md(size_t nz, size_t ny, size_t nx, int dims) {
  MdGrid g;
  if (!md_grid(nz, ny, nx, dims, &g)) return 0;
  return size_t(kHdr + align16(g.nb) + 128 * g.nb);   // 32-word garbage bound, as cuszp_max_compressed_bytes
}

size_t cuszp_workspace_bytes_md(size_t nz, size_t ny, size_t nx, int dims) {
  MdGrid g;
  if (!md_grid(nz, ny, nx, dims, &g)) return 0;
  const uint64_t t = (g.nb + kTileBlocks - 1) / kTileBlocks;
  return size_t(kWsCtrlBytes + 8 * (t > 0 ? t : 1));
}

int cuszp_compress_md(const float* d_in, size_t nz, size_t ny, size_t nx, int dims, float eb, int mode, void* d_out,
                      size_t out_capacity, unsigned long long* d_out_bytes, void* d_ws, size_t ws_bytes,
                      void* stream) {
  MdGrid g;
  if (d_in == nullptr || d_out == nullptr || d_ws == nullptr || !md_grid(nz, ny, nx, dims, &g)) return CUSZP_EINVAL;
  if ((reinterpret_cast<uintptr_t>(d_in) & 15u) || (reinterpret_cast<uintptr_t>(d_out) & 15u) ||
      (reinterpret_cast<uintptr_t>(d_ws) & 15u))
    return CUSZP_EINVAL;
  const size_t n = nz * ny * nx;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (out_capacity < cuszp_max_compressed_bytes_md(nz, ny, nx, dims) ||
      ws_bytes < cuszp_workspace_bytes_md(nz, ny, nx, dims))
    return CUSZP_ENOSPACE;
  if (mode == CUSZP_ABS) {
    if (!eb_is_normal(eb)) return CUSZP_EINVAL;
    return launch_compress(d_in, n, CUSZP_ABS, eb, nullptr, 0, d_out, out_capacity, d_out_bytes, d_ws, ws_bytes, s,
                           kL, 1, &g);
  }
  if (mode == CUSZP_REL) {
    if (!(eb > 0.0f) || !(eb - eb == 0.0f)) return CUSZP_EINVAL;
    const int st = cuszp_range(d_in, n, nullptr, d_ws, ws_bytes, stream);
    if (st != CUSZP_OK) return st;
    return launch_compress(d_in, n, CUSZP_REL, eb, static_cast<const WsCtrl*>(d_ws)->minmax, 1, d_out,
                           out_capacity, d_out_bytes, d_ws, ws_bytes, s, kL, 1, &g);
  }
  return CUSZP_EINVAL;
}

int cuszp_decompress_md(const void* d_in, size_t in_bytes, float* d_out, size_t nz, size_t ny, size_t nx, int dims,
                        void* d_ws, size_t ws_bytes, void* stream) {
  MdGrid g;
  if (d_in == nullptr || d_out == nullptr || d_ws == nullptr || !md_grid(nz, ny, nx, dims, &g)) return CUSZP_EINVAL;
  if ((reinterpret_cast<uintptr_t>(d_in) & 15u) || (reinterpret_cast<uintptr_t>(d_out) & 15u) ||
      (reinterpret_cast<uintptr_t>(d_ws) & 15u))
    return CUSZP_EINVAL;
  if (ws_bytes < cuszp_workspace_bytes_md(nz, ny, nx, dims)) return CUSZP_ENOSPACE;
  DeviceInfo di;
  if (device_info(&di) != CUSZP_OK) return CUSZP_ECUDA;
  DecompressArgs a;
  a.in = static_cast<const uint8_t*>(d_in);
  a.in_bytes = in_bytes;
  a.out = d_out;
  a.n = nz * ny * nx;
  a.nb = g.nb;
  a.num_tiles = uint32_t((g.nb + kTileBlocks - 1) / kTileBlocks);
  a.ws = static_cast<WsCtrl*>(d_ws);
  a.status = reinterpret_cast<uint64_t*>(static_cast<uint8_t*>(d_ws) + kWsCtrlBytes);
  a.status_cap = status_capacity(ws_bytes);
  a.trace = g_trace;
  a.dims = dims;
  a.nz = g.nz;
  a.ny = g.ny;
  a.nx = g.nx;
  a.nby = g.nby;
  a.nbx = g.nbx;
  a.fd_nbx = FastDiv(uint32_t(g.nbx));
  a.fd_nby = FastDiv(uint32_t(g.nby));
  const int occ = di.occ_d[2];
  uint64_t grid = uint64_t(di.sms) * uint64_t(occ > 0 ? occ : 1);
  if (g_grid_decompress > 0) grid = uint64_t(g_grid_decompress);
  a.chunk_tiles = decompress_chunk_tiles(a.num_tiles, grid);
  if (grid > a.num_tiles) grid = a.num_tiles;
  if (grid < 1) grid = 1;
  return decompress_launch(32, 1, unsigned(grid), a, static_cast<cudaStream_t>(stream)) == cudaSuccess ? CUSZP_OK
                                                                                                    : CUSZP_ECUDA;
}

int cuszp_last_status(const void* d_ws, void* stream) {
  if (d_ws == nullptr) return CUSZP_EINVAL;
  uint32_t st = 0;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (cudaMemcpyAsync(&st, &static_cast<const WsCtrl*>(d_ws)->last_status, 4, cudaMemcpyDeviceToHost, s) !=
          cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return CUSZP_ECUDA;
  return int(st);
}

int cuszp_read_header(const void* d_stream, cuszp_header* h_hdr, void* stream) {
  if (d_stream == nullptr || h_hdr == nullptr) return CUSZP_EINVAL;
  static_assert(sizeof(cuszp_header) == 32, "header layout");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (cudaMemcpyAsync(h_hdr, d_stream, 32, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return CUSZP_ECUDA;
  return CUSZP_OK;
}

int cuszp_compress_host(const float* h_in, size_t n, float eb, int mode, void* h_out, size_t out_capacity,
                        size_t* h_out_bytes, float* d_in_scratch, void* d_out_scratch, void* d_ws,
                        size_t ws_bytes, void* stream) {
  if ((n > 0 && (h_in == nullptr || d_in_scratch == nullptr)) || h_out == nullptr || h_out_bytes == nullptr ||
      d_out_scratch == nullptr)
    return CUSZP_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (n > 0 && cudaMemcpyAsync(d_in_scratch, h_in, n * sizeof(float), cudaMemcpyHostToDevice, s) != cudaSuccess)
    return CUSZP_ECUDA;
  // the exact length lands in the workspace's pad area (device u64)
  unsigned long long* d_len =
      reinterpret_cast<unsigned long long*>(&static_cast<WsCtrl*>(d_ws)->pad[2]);
  int st = cuszp_compress(d_in_scratch, n, eb, mode, d_out_scratch, cuszp_max_compressed_bytes(n), d_len, d_ws,
                          ws_bytes, stream);
  if (st != CUSZP_OK) return st;
  unsigned long long len = 0;
  if (cudaMemcpyAsync(&len, d_len, 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return CUSZP_ECUDA;
  if (len > out_capacity) return CUSZP_ENOSPACE;
  if (cudaMemcpyAsync(h_out, d_out_scratch, size_t(len), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return CUSZP_ECUDA;
  *h_out_bytes = size_t(len);
  return CUSZP_OK;
}

int cuszp_decompress_host(const void* h_in, size_t in_bytes, float* h_out, size_t n, void* d_in_scratch,
                          float* d_out_scratch, void* d_ws, size_t ws_bytes, void* stream) {
  if (h_in == nullptr || d_in_scratch == nullptr || (n > 0 && (h_out == nullptr || d_out_scratch == nullptr)))
    return CUSZP_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (cudaMemcpyAsync(d_in_scratch, h_in, in_bytes, cudaMemcpyHostToDevice, s) != cudaSuccess)
    return CUSZP_ECUDA;
  int st = cuszp_decompress(d_in_scratch, in_bytes, d_out_scratch, n, d_ws, ws_bytes, stream);
  if (st != CUSZP_OK) return st;
  if (n > 0 && cudaMemcpyAsync(h_out, d_out_scratch, n * sizeof(float), cudaMemcpyDeviceToHost, s) != cudaSuccess)
    return CUSZP_ECUDA;
  if (cudaStreamSynchronize(s) != cudaSuccess) return CUSZP_ECUDA;
  return CUSZP_OK;
}

namespace {
// device-visible address of a host-mapped pinned buffer (nullptr if not mapped)
void* mapped(const void* h) {
  void* d = nullptr;
  if (h == nullptr || cudaHostGetDevicePointer(&d, const_cast<void*>(h), 0) != cudaSuccess) {
    cudaGetLastError();   // clear the sticky-free error state of the failed query
    return nullptr;
  }
  return d;
}
}  // namespace

int cuszp_compress_host_async(const float* h_in, size_t n, float eb, int mode, void* h_out, size_t out_capacity,
                              unsigned long long* h_out_bytes, float* d_in_scratch, void* d_out_scratch, void* d_ws,
                              size_t ws_bytes, void* stream) {
  if ((n > 0 && (h_in == nullptr || d_in_scratch == nullptr)) || d_out_scratch == nullptr || d_ws == nullptr)
    return CUSZP_EINVAL;
  // every check precedes the first launch: the copy kernel moves
  // 16-byte words into h_out and an 8-byte length into h_out_bytes
  if (misaligned(h_out, 16) || misaligned(h_out_bytes, 8) || misaligned(d_in_scratch, 16) ||
      misaligned(d_out_scratch, 16) || misaligned(d_ws, 16))
    return CUSZP_EINVAL;
  if (out_capacity < cuszp_max_compressed_bytes(n)) return CUSZP_ENOSPACE;
  if (ws_bytes < cuszp_workspace_bytes(n)) return CUSZP_ENOSPACE;
  if (mode == CUSZP_ABS ? !eb_is_normal(eb) : (mode != CUSZP_REL || !(eb > 0.0f) || !(eb - eb == 0.0f)))
    return CUSZP_EINVAL;
  void* out_dev = mapped(h_out);
  unsigned long long* len_dev = static_cast<unsigned long long*>(mapped(h_out_bytes));
  if (out_dev == nullptr || len_dev == nullptr) return CUSZP_EINVAL;
  DeviceInfo di;
  if (device_info(&di) != CUSZP_OK) return CUSZP_ECUDA;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (n > 0 && cudaMemcpyAsync(d_in_scratch, h_in, n * sizeof(float), cudaMemcpyHostToDevice, s) != cudaSuccess)
    return CUSZP_ECUDA;
  unsigned long long* d_len = reinterpret_cast<unsigned long long*>(&static_cast<WsCtrl*>(d_ws)->pad[2]);
  int st = cuszp_compress(d_in_scratch, n, eb, mode, d_out_scratch, cuszp_max_compressed_bytes(n), d_len, d_ws,
                          ws_bytes, stream);
  if (st != CUSZP_OK) return st;
  // exactly the stream's bytes cross the link; its length lands in *h_out_bytes
  return launch_copy_len(out_dev, d_out_scratch, d_len, out_capacity, len_dev, di.sms, s);
}

int cuszp_decompress_host_async(const void* h_in, size_t in_capacity, float* h_out, size_t n, void* d_in_scratch,
                                float* d_out_scratch, void* d_ws, size_t ws_bytes, void* stream) {
  if (h_in == nullptr || d_in_scratch == nullptr || d_ws == nullptr ||
      (n > 0 && (h_out == nullptr || d_out_scratch == nullptr)))
    return CUSZP_EINVAL;
  if (in_capacity < size_t(kHdr)) return CUSZP_EINVAL;
  // every check precedes the first launch: the copy kernel reads
  // 16-byte words of h_in and writes them into d_in_scratch
  if (misaligned(h_in, 16) || misaligned(d_in_scratch, 16) || misaligned(d_out_scratch, 16) || misaligned(d_ws, 16))
    return CUSZP_EINVAL;
  if (ws_bytes < cuszp_workspace_bytes(n)) return CUSZP_ENOSPACE;
  const void* in_dev = mapped(h_in);
  if (in_dev == nullptr) return CUSZP_EINVAL;
  DeviceInfo di;
  if (device_info(&di) != CUSZP_OK) return CUSZP_ECUDA;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  unsigned long long* d_len = reinterpret_cast<unsigned long long*>(&static_cast<WsCtrl*>(d_ws)->pad[4]);
  int st = launch_stream_len(in_dev, n, d_len, s);                        // length from the stream's header
  if (st == CUSZP_OK) st = launch_copy_len(d_in_scratch, in_dev, d_len, in_capacity, nullptr, di.sms, s);
  if (st == CUSZP_OK) st = cuszp_decompress(d_in_scratch, in_capacity, d_out_scratch, n, d_ws, ws_bytes, stream);
  if (st != CUSZP_OK) return st;
  if (n > 0 && cudaMemcpyAsync(h_out, d_out_scratch, n * sizeof(float), cudaMemcpyDeviceToHost, s) != cudaSuccess)
    return CUSZP_ECUDA;
  return CUSZP_OK;
}

int cuszp_container_put(const void* d_shard, const void* d_header, unsigned P, unsigned p, void* d_container,
                        int write_header, void* stream) {
  if (d_shard == nullptr || d_header == nullptr || d_container == nullptr || P == 0 || p >= P) return CUSZP_EINVAL;
  if (misaligned(d_shard, 16) || misaligned(d_container, 16) || misaligned(d_header, 8)) return CUSZP_EINVAL;
  DeviceInfo di;
  if (device_info(&di) != CUSZP_OK) return CUSZP_ECUDA;
  return launch_container_put(d_shard, d_header, P, p, d_container, write_header, di.sms,
                              static_cast<cudaStream_t>(stream));
}

const char* cuszp_status_string(int status) {
  switch (status) {
    case CUSZP_OK: return "CUSZP_OK";
    case CUSZP_EINVAL: return "CUSZP_EINVAL";
    case CUSZP_ECUDA: return "CUSZP_ECUDA";
    case CUSZP_ERANGE: return "CUSZP_ERANGE";
    case CUSZP_ECORRUPT: return "CUSZP_ECORRUPT";
    case CUSZP_ENOSPACE: return "CUSZP_ENOSPACE";
    default: return "CUSZP_UNKNOWN";
  }
}

int cuszp_version(void) { return CUSZP_VERSION * 100 + 1; }

// diagnostics only (not declared in include/cuszp.h)
void cuszp_debug_set_trace(void* d_trace) { g_trace = static_cast<uint64_t*>(d_trace); }
void cuszp_debug_set_grid(int compress_grid, int decompress_grid) {
  g_grid_compress = compress_grid;
  g_grid_decompress = decompress_grid;
}
int cuszp_debug_occupancy(int* out4) {
  DeviceInfo di;
  if (device_info(&di) != CUSZP_OK) return CUSZP_ECUDA;
  out4[0] = di.sms;
  out4[1] = di.occ_compress;
  out4[2] = di.occ_decompress;
  out4[3] = di.occ_range;
  return CUSZP_OK;
}

}  // extern "C"
