/*
 * cuszp_oracle.cpp -- plain single-threaded C++17 oracle of the cuSZp
 * compress / decompress path.  TEST INFRASTRUCTURE ONLY (see header).
 *
 * Written from the paper text, step by step, in the paper's order and
 * notation (d_i data, r_i quantisation integers, l_i Lorenzo integers,
 * F_k fixed length, CmpL_k block bytes).  No blocking, fusion or
 * reordering beyond what the paper states.  Readings of ambiguous or
 * garbled passages are DESIGN.md sec. 3, items R1..R12, cited as "R#".
 *
 * Build (kept deliberately plain; see __graft_entry__.build()):
 *   g++ -std=c++17 -O2 -ffp-contract=off -fno-fast-math -shared -fPIC
 * -ffp-contract=off keeps every float op a separately rounded IEEE op;
 * the one fused multiply-add of the op sequence is an explicit fmaf().
 */
#include "cuszp_oracle.h"

#include <cfenv>
#include <cmath>
#include <cstring>
#include <vector>

int prequantize_guarded(const float* x, size_t n, float eb_abs, int32_t* q, float guard);
void block_lorenzo_order(const int32_t* q, size_t nb, int L, int order, int32_t* l);

namespace {

const int L = 32;                     /* default block length, R1 */
const int MAX_L = 128;                /* block lengths 8..128 */

bool valid_block_len(int Lb) { return Lb == 8 || Lb == 16 || Lb == 32 || Lb == 64 || Lb == 128; }
int log2_of(int Lb) { int k = 0; while ((1 << k) < Lb) ++k; return k; }
const int HEADER_BYTES = 32;          /* R10 */
const float GUARD = 4194304.0f;       /* 2^22, R5 */
const float GUARD2 = 2097152.0f;      /* 2^21: 2-layer Lorenzo keeps |l| <= 2^23 (R17) */
const int MAX_F = 24;                 /* consequence of the guard, R5 */

uint64_t align16(uint64_t v) { return (v + 15u) & ~uint64_t(15); }

void put_u64(uint8_t* p, uint64_t v) { for (int i = 0; i < 8; ++i) p[i] = uint8_t(v >> (8 * i)); }
uint64_t get_u64(const uint8_t* p) { uint64_t v = 0; for (int i = 0; i < 8; ++i) v |= uint64_t(p[i]) << (8 * i); return v; }
void put_u32(uint8_t* p, uint32_t v) { for (int i = 0; i < 4; ++i) p[i] = uint8_t(v >> (8 * i)); }
uint32_t get_u32(const uint8_t* p) { uint32_t v = 0; for (int i = 0; i < 4; ++i) v |= uint32_t(p[i]) << (8 * i); return v; }
void put_f32(uint8_t* p, float f) { uint32_t u; std::memcpy(&u, &f, 4); put_u32(p, u); }
float get_f32(const uint8_t* p) { uint32_t u = get_u32(p); float f; std::memcpy(&f, &u, 4); return f; }

/* An absolute error bound is usable when eb and 2eb are positive, finite
 * and normal (R5): 1/(2eb) is then finite. */
bool eb_usable(float eb) {
  if (!(eb >= 1.17549435e-38f)) return false;   /* FLT_MIN; rejects NaN, 0, <0 */
  float two_eb = eb + eb;
  return std::isfinite(two_eb);
}

/* Stream header, R10:
 *  0 'CSZP' | 4 version=1 | 5 mode | 6 status | 7 log2(L)=5 | 8 u64 n |
 * 16 f32 eb_abs | 20 f32 eb_in | 24 u64 payload_bytes                    */
void write_header(uint8_t* out, uint64_t n, int mode, int status, float eb_abs,
                  float eb_in, uint64_t payload_bytes, int Lb) {
  out[0] = 'C'; out[1] = 'S'; out[2] = 'Z'; out[3] = 'P';
  out[4] = 1; out[5] = uint8_t(mode); out[6] = uint8_t(status); out[7] = uint8_t(log2_of(Lb));
  put_u64(out + 8, n);
  put_f32(out + 16, eb_abs);
  put_f32(out + 20, eb_in);
  put_u64(out + 24, payload_bytes);
}

uint64_t encode_and_place(const int32_t* l, uint64_t nb, int L, uint8_t* out);

/* Compression of x[0..n) with a resolved absolute bound eb_abs (sec 3.1,
 * Fig 2): Quantisation and Prediction -> Fixed-length Encoding ->
 * Global Synchronization -> Block Bit-shuffle. */
int compress_with_eb(const float* x, uint64_t n, float eb_abs, float eb_in, int mode,
                     uint8_t* out, uint64_t cap, uint64_t* out_bytes, int L, int order = 1) {
  mode |= (order == 2) ? 0x10 : 0;                      /* header: predictor order (R17) */
  const uint64_t nb = (n + L - 1) / L;                  /* number of blocks N */
  if (cap < oracle_max_compressed_bytes_L(n, L)) return ORACLE_ENOSPACE;
  std::memset(out, 0, size_t(HEADER_BYTES + align16(nb)));

  if (n == 0) {                                         /* R11 */
    write_header(out, 0, mode, ORACLE_OK, eb_abs, eb_in, 0, L);
    *out_bytes = HEADER_BYTES;
    return ORACLE_OK;
  }
  if (!eb_usable(eb_abs)) {                             /* R5 */
    write_header(out, n, mode, ORACLE_ERANGE, eb_abs, eb_in, 0, L);
    *out_bytes = HEADER_BYTES + align16(nb);
    return ORACLE_ERANGE;
  }

  /* (1) Pre-quantisation, the only lossy step. */
  std::vector<int32_t> r(static_cast<size_t>(nb * L), 0);            /* zero pad, R8 */
  if (prequantize_guarded(x, size_t(n), eb_abs, r.data(), order == 2 ? GUARD2 : GUARD) != ORACLE_OK) {
    write_header(out, n, mode, ORACLE_ERANGE, eb_abs, eb_in, 0, L);
    *out_bytes = HEADER_BYTES + align16(nb);
    return ORACLE_ERANGE;
  }

  /* (1') Lorenzo prediction inside each block. */
  std::vector<int32_t> l(static_cast<size_t>(nb * L));
  block_lorenzo_order(r.data(), size_t(nb), L, order, l.data());

  const uint64_t payload_bytes = encode_and_place(l.data(), nb, L, out);
  write_header(out, n, mode, ORACLE_OK, eb_abs, eb_in, payload_bytes, L);
  *out_bytes = HEADER_BYTES + align16(nb) + payload_bytes;
  return ORACLE_OK;
}

/* Steps (2)-(4) of compression for nb blocks of Lorenzo integers l[nb*L]:
 * the F bytes go to out[32..], the payloads to their synchronised offsets;
 * returns the payload bytes (the sum of CmpL). */
uint64_t encode_and_place(const int32_t* l, uint64_t nb, int L, uint8_t* out) {
  /* (2) Fixed-length encoding: F_k and CmpL_k per block,
   *     giving the BlockOffsetArray. */
  std::vector<std::vector<uint8_t>> encoded(static_cast<size_t>(nb));
  std::vector<uint64_t> block_offset(static_cast<size_t>(nb));
  uint8_t* fixed_length = out + HEADER_BYTES;          /* Fig 12 part 1 */
  for (uint64_t k = 0; k < nb; ++k) {
    uint8_t buf[(MAX_L / 8) * (MAX_F + 1)];
    int F = oracle_encode_block_L(&l[size_t(k * L)], L, buf);
    fixed_length[k] = uint8_t(F);
    block_offset[k] = oracle_block_bytes(F, L);
    encoded[k].assign(buf, buf + block_offset[k]);
  }

  /* (3) Global synchronisation = exclusive prefix sum (Eq 3). */
  std::vector<uint64_t> sync_offset(static_cast<size_t>(nb));
  oracle_exclusive_scan(block_offset.data(), size_t(nb), sync_offset.data());
  const uint64_t payload_bytes = sync_offset[nb - 1] + block_offset[nb - 1];

  /* (4) Block bit-shuffled bytes placed at the synchronised offsets
   *     (Fig 12 part 2). */
  const uint64_t p0 = HEADER_BYTES + align16(nb);
  for (uint64_t k = 0; k < nb; ++k)
    if (block_offset[k] > 0)
      std::memcpy(out + p0 + sync_offset[k], encoded[k].data(), size_t(block_offset[k]));
  return payload_bytes;
}

}  // namespace

extern "C" {

void oracle_value_range(const float* x, size_t n, float* mn, float* mx) {
  /* r = max value - min value of the dataset.  A NaN anywhere
   * makes the range undefined: both ends are reported as NaN (R5). */
  float lo = INFINITY, hi = -INFINITY;
  bool has_nan = false;
  for (size_t i = 0; i < n; ++i) {
    if (std::isnan(x[i])) { has_nan = true; continue; }
    if (x[i] < lo) lo = x[i];
    if (x[i] > hi) hi = x[i];
  }
  *mn = has_nan ? NAN : lo;
  *mx = has_nan ? NAN : hi;
}

int oracle_prequantize(const float* x, size_t n, float eb_abs, int32_t* q) {
  return prequantize_guarded(x, n, eb_abs, q, GUARD);
}

}  // extern "C"

/* R2 with the guard of the predictor order (R5 / R17). */
int prequantize_guarded(const float* x, size_t n, float eb_abs, int32_t* q, float guard) {
  /* r_i = round(d_i / 2eb), guaranteeing |r_i * 2eb - d_i| <= eb.
   * fp32 op sequence R2 (shared by definition, not by code, with the GPU):
   *   two_eb = eb + eb; recip = 1 / two_eb           (fp32, once)
   *   r0  = nearest integer (ties to even) to the EXACT product d * recip
   *         -- one rounding; the product of two floats is exact in double
   *   guard: |r0| < 2^22, else ERANGE (R5; NaN and Inf fail it)
   *   res = fmaf(-r0, two_eb, d)   -- exact, see DESIGN R2
   *   r   = r0 + (res > eb) - (res < -eb)   -> |d - r*2eb| <= eb exactly  */
  std::fesetround(FE_TONEAREST);
  const float two_eb = eb_abs + eb_abs;
  const float recip = 1.0f / two_eb;
  for (size_t i = 0; i < n; ++i) {
    const double p = double(x[i]) * double(recip);      /* exact */
    const double r0d = std::nearbyint(p);
    if (!(std::fabs(r0d) < double(guard))) return ORACLE_ERANGE;
    const float r0 = float(r0d);                         /* exact, |r0| < 2^22 */
    const float res = std::fmaf(-r0, two_eb, x[i]);
    int32_t r = int32_t(r0);
    if (res > eb_abs) r += 1;
    else if (res < -eb_abs) r -= 1;
    q[i] = r;
  }
  return ORACLE_OK;
}

/* 2-layer 1D Lorenzo inside each block (R17):
 * l_i = r_i - 2 r_{i-1} + r_{i-2}, r_{-1} = r_{-2} = 0 at every block start. */
void block_lorenzo_order(const int32_t* q, size_t nb, int L, int order, int32_t* l) {
  if (order != 2) { oracle_block_lorenzo_L(q, nb, L, l); return; }
  for (size_t k = 0; k < nb; ++k) {
    const int32_t* r = q + k * L;
    int32_t* lk = l + k * L;
    for (int i = 0; i < L; ++i) {
      const int32_t p1 = (i >= 1) ? r[i - 1] : 0;
      const int32_t p2 = (i >= 2) ? r[i - 2] : 0;
      lk[i] = r[i] - 2 * p1 + p2;
    }
  }
}

extern "C" {

void oracle_block_lorenzo(const int32_t* q, size_t nb, int32_t* l) {
  oracle_block_lorenzo_L(q, nb, L, l);
}

void oracle_block_lorenzo_L(const int32_t* q, size_t nb, int L, int32_t* l) {
  /* l_i = r_i - r_{i-1}, r_{i-1} = 0 for the first integer of each block
   * (P:525-529): the linear recurrence never crosses a block. */
  for (size_t k = 0; k < nb; ++k) {
    const int32_t* r = q + k * L;
    int32_t* lk = l + k * L;
    for (int i = 0; i < L; ++i) {
      const int32_t prev = (i == 0) ? 0 : r[i - 1];
      lk[i] = r[i] - prev;
    }
  }
}

int oracle_bit_length(uint32_t m) {
  /* "the position of the last non-zero bit of this maximum integer"
   * (P:566-568): 11 -> 4, 134 -> 8. */
  int F = 0;
  while (m != 0) { ++F; m >>= 1; }
  return F;
}

uint64_t oracle_block_bytes(int F, int Lb) {
  /* Eq 2: CmpL_k = (F_k + 1) * L / 8; a zero block stores nothing but
   * its fixed-length byte (R6). */
  if (F == 0) return 0;
  return uint64_t(F + 1) * uint64_t(Lb) / 8;
}

void oracle_exclusive_scan(const uint64_t* cmpl, size_t k, uint64_t* sync_off) {
  /* Eq 3: SyncOffsetArray = {0, CmpL_0, CmpL_0 + CmpL_1, ...}. */
  uint64_t s = 0;
  for (size_t i = 0; i < k; ++i) { sync_off[i] = s; s += cmpl[i]; }
}

int oracle_encode_block(const int32_t l[32], uint8_t* out) { return oracle_encode_block_L(l, L, out); }

int oracle_encode_block_L(const int32_t* l, int L, uint8_t* out) {
  /* Sign map: bit 0 for positive, 1 otherwise; integer 0 -> bit 0 (R7).
   * L/8 bytes; element j -> byte j/8, bit j%8 (R9). */
  uint8_t sign_map[MAX_L / 8] = {0};
  uint32_t mag[MAX_L];
  uint32_t max_abs = 0;
  for (int j = 0; j < L; ++j) {
    if (l[j] < 0) sign_map[j / 8] |= uint8_t(1u << (j % 8));
    mag[j] = (l[j] < 0) ? uint32_t(-int64_t(l[j])) : uint32_t(l[j]);
    if (mag[j] > max_abs) max_abs = mag[j];
  }
  /* Fixed length F = bit length of the block maximum. */
  const int F = oracle_bit_length(max_abs);
  if (F == 0) return 0;                                 /* zero block */
  /* Block bit-shuffle: bit k of every |l_j| goes to the k-th
   * group of L/8 bytes, after the sign map (R9). */
  std::memcpy(out, sign_map, L / 8);
  for (int k = 0; k < F; ++k) {
    uint8_t* plane = out + (L / 8) * (1 + k);
    for (int b = 0; b < L / 8; ++b) plane[b] = 0;
    for (int j = 0; j < L; ++j)
      if ((mag[j] >> k) & 1u) plane[j / 8] |= uint8_t(1u << (j % 8));
  }
  return F;
}

void oracle_decode_block(const uint8_t* payload, int F, int32_t l[32]) {
  oracle_decode_block_L(payload, F, L, l);
}

void oracle_decode_block_L(const uint8_t* payload, int F, int L, int32_t* l) {
  if (F == 0) { for (int j = 0; j < L; ++j) l[j] = 0; return; }
  for (int j = 0; j < L; ++j) {
    uint32_t mag = 0;
    for (int k = 0; k < F; ++k) {
      const uint8_t* plane = payload + (L / 8) * (1 + k);
      if ((plane[j / 8] >> (j % 8)) & 1u) mag |= 1u << k;
    }
    const bool negative = (payload[j / 8] >> (j % 8)) & 1u;
    l[j] = negative ? -int32_t(mag) : int32_t(mag);
  }
}

uint64_t oracle_max_compressed_bytes(uint64_t n) { return oracle_max_compressed_bytes_L(n, L); }

uint64_t oracle_max_compressed_bytes_L(uint64_t n, int L) {
  const uint64_t nb = (n + L - 1) / L;
  return HEADER_BYTES + align16(nb) + uint64_t(L / 8) * uint64_t(MAX_F + 1) * nb;
}

int oracle_compress(const float* x, uint64_t n, float eb, int mode,
                    uint8_t* out, uint64_t cap, uint64_t* out_bytes) {
  return oracle_compress_L(x, n, eb, mode, L, out, cap, out_bytes);
}

int oracle_compress_L(const float* x, uint64_t n, float eb, int mode, int L,
                      uint8_t* out, uint64_t cap, uint64_t* out_bytes) {
  return oracle_compress_ex(x, n, eb, mode, L, 1, out, cap, out_bytes);
}

int oracle_compress_ex(const float* x, uint64_t n, float eb, int mode, int L, int order,
                       uint8_t* out, uint64_t cap, uint64_t* out_bytes) {
  if ((n > 0 && x == nullptr) || out == nullptr || out_bytes == nullptr || !valid_block_len(L) ||
      (order != 1 && order != 2))
    return ORACLE_EINVAL;
  if (mode == 0) {                                      /* ABS: eb = delta */
    if (!eb_usable(eb)) return ORACLE_EINVAL;
    return compress_with_eb(x, n, eb, eb, 0, out, cap, out_bytes, L, order);
  }
  if (mode == 1) {                                      /* REL: eb = lambda * r */
    if (!(eb > 0.0f) || !std::isfinite(eb)) return ORACLE_EINVAL;
    if (n == 0) return compress_with_eb(x, 0, 0.0f, eb, 1, out, cap, out_bytes, L, order);
    float mn, mx;
    oracle_value_range(x, size_t(n), &mn, &mx);
    const float range = mx - mn;                        /* R3: fp32 */
    const float eb_abs = eb * range;
    return compress_with_eb(x, n, eb_abs, eb, 1, out, cap, out_bytes, L, order);
  }
  return ORACLE_EINVAL;
}

int oracle_compress_minmax(const float* x, uint64_t n, float lambda,
                           const float* minmax, int n_pairs,
                           uint8_t* out, uint64_t cap, uint64_t* out_bytes) {
  return oracle_compress_minmax_L(x, n, lambda, minmax, n_pairs, L, out, cap, out_bytes);
}

int oracle_compress_minmax_L(const float* x, uint64_t n, float lambda,
                             const float* minmax, int n_pairs, int L,
                             uint8_t* out, uint64_t cap, uint64_t* out_bytes) {
  if ((n > 0 && x == nullptr) || out == nullptr || out_bytes == nullptr ||
      minmax == nullptr || n_pairs <= 0 || !valid_block_len(L)) return ORACLE_EINVAL;
  if (!(lambda > 0.0f) || !std::isfinite(lambda)) return ORACLE_EINVAL;
  float mn = minmax[0], mx = minmax[1];
  for (int p = 1; p < n_pairs; ++p) {
    if (minmax[2 * p] < mn) mn = minmax[2 * p];
    if (minmax[2 * p + 1] > mx) mx = minmax[2 * p + 1];
  }
  const float range = mx - mn;
  const float eb_abs = lambda * range;
  return compress_with_eb(x, n, eb_abs, lambda, 1, out, cap, out_bytes, L);
}

int oracle_decompress(const uint8_t* in, uint64_t in_bytes, float* out, uint64_t n) {
  /* Sec 3.2 / Fig 3: read the fixed lengths, rebuild CmpL (Eq 2), the same
   * global synchronisation (Eq 3), then reverse bit-shuffle, fixed-length
   * encoding and quantisation + prediction. */
  if (in == nullptr || (n > 0 && out == nullptr)) return ORACLE_EINVAL;
  if (in_bytes < uint64_t(HEADER_BYTES)) return ORACLE_ECORRUPT;
  if (!(in[0] == 'C' && in[1] == 'S' && in[2] == 'Z' && in[3] == 'P') ||
      in[4] != 1 || in[7] < 3 || in[7] > 7) return ORACLE_ECORRUPT;
  const int L = 1 << in[7];                             /* block length from the header */
  const int order = (in[5] & 0x10) ? 2 : 1;             /* predictor order from the header (R17) */
  if (in[6] != ORACLE_OK) return in[6] == ORACLE_ERANGE ? ORACLE_ERANGE : ORACLE_ECORRUPT;
  if (get_u64(in + 8) != n) return ORACLE_EINVAL;
  if (n == 0) return ORACLE_OK;
  const float eb_abs = get_f32(in + 16);
  const uint64_t payload_bytes = get_u64(in + 24);
  const uint64_t nb = (n + L - 1) / L;
  const uint64_t p0 = HEADER_BYTES + align16(nb);
  if (in_bytes < p0) return ORACLE_ECORRUPT;
  if (!eb_usable(eb_abs)) return ORACLE_ECORRUPT;

  const uint8_t* fixed_length = in + HEADER_BYTES;
  std::vector<uint64_t> block_offset(static_cast<size_t>(nb));
  for (uint64_t k = 0; k < nb; ++k) {
    if (fixed_length[k] > MAX_F) return ORACLE_ECORRUPT;
    block_offset[k] = oracle_block_bytes(fixed_length[k], L);
  }
  std::vector<uint64_t> sync_offset(static_cast<size_t>(nb));
  oracle_exclusive_scan(block_offset.data(), size_t(nb), sync_offset.data());
  const uint64_t total = sync_offset[nb - 1] + block_offset[nb - 1];
  if (total != payload_bytes || in_bytes < p0 + total) return ORACLE_ECORRUPT;

  const float two_eb = eb_abs + eb_abs;
  for (uint64_t k = 0; k < nb; ++k) {
    int32_t l[MAX_L];
    oracle_decode_block_L(in + p0 + sync_offset[k], fixed_length[k], L, l);
    /* reverse Lorenzo: r_i = r_{i-1} + l_i inside the block (order 2:
     * r_i = l_i + 2 r_{i-1} - r_{i-2}) */
    int32_t r = 0, r1 = 0, r2 = 0;
    for (int i = 0; i < L; ++i) {
      if (order == 2) {
        r = l[i] + 2 * r1 - r2;
        r2 = r1;
        r1 = r;
      } else {
        r += l[i];
      }
      const uint64_t idx = k * L + uint64_t(i);
      /* d'_i = r_i * 2eb */
      if (idx < n) out[idx] = float(r) * two_eb;
    }
  }
  return ORACLE_OK;
}

/* ---- multi-dimensional Lorenzo inside blocks (DESIGN R18) ---- */

namespace {

/* block box (bz, by, bx) of the dims-D predictor: 1x4x8 (2D), 2x4x4 (3D) */
void md_box(int dims, int* bz, int* by, int* bx) {
  *bz = (dims == 3) ? 2 : 1;
  *by = 4;
  *bx = (dims == 3) ? 4 : 8;
}

uint64_t ceil_div(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

bool md_args_ok(uint64_t nz, uint64_t ny, uint64_t nx, int dims) {
  return (dims == 2 || dims == 3) && nz > 0 && ny > 0 && nx > 0;
}

}  // namespace

uint64_t oracle_num_blocks_md(uint64_t nz, uint64_t ny, uint64_t nx, int dims) {
  int bz, by, bx;
  md_box(dims, &bz, &by, &bx);
  return ceil_div(nz, bz) * ceil_div(ny, by) * ceil_div(nx, bx);
}

uint64_t oracle_max_compressed_bytes_md(uint64_t nz, uint64_t ny, uint64_t nx, int dims) {
  const uint64_t nb = oracle_num_blocks_md(nz, ny, nx, dims);
  return HEADER_BYTES + align16(nb) + uint64_t(L / 8) * uint64_t(MAX_F + 1) * nb;
}

void oracle_block_lorenzo_md(const int32_t r[32], int dims, int32_t l[32]) {
  /* The Lorenzo predictor (ref [14]) restricted to the block: every
   * neighbour outside the block counts as 0. */
  int bz, by, bx;
  md_box(dims, &bz, &by, &bx);
  auto at = [&](int z, int y, int x) -> int32_t {
    if (z < 0 || y < 0 || x < 0) return 0;
    return r[(z * by + y) * bx + x];
  };
  for (int z = 0; z < bz; ++z)
    for (int y = 0; y < by; ++y)
      for (int x = 0; x < bx; ++x) {
        int32_t pred;
        if (dims == 2)
          pred = at(z, y, x - 1) + at(z, y - 1, x) - at(z, y - 1, x - 1);
        else
          pred = at(z, y, x - 1) + at(z, y - 1, x) + at(z - 1, y, x)
                 - at(z, y - 1, x - 1) - at(z - 1, y, x - 1) - at(z - 1, y - 1, x)
                 + at(z - 1, y - 1, x - 1);
        l[(z * by + y) * bx + x] = at(z, y, x) - pred;
      }
}

int oracle_compress_md(const float* x, uint64_t nz, uint64_t ny, uint64_t nx, int dims, float eb,
                       int mode, uint8_t* out, uint64_t cap, uint64_t* out_bytes) {
  if (x == nullptr || out == nullptr || out_bytes == nullptr || !md_args_ok(nz, ny, nx, dims))
    return ORACLE_EINVAL;
  const uint64_t n = nz * ny * nx;
  const uint64_t nb = oracle_num_blocks_md(nz, ny, nx, dims);
  if (cap < oracle_max_compressed_bytes_md(nz, ny, nx, dims)) return ORACLE_ENOSPACE;
  const int mode_byte = mode | ((dims - 1) << 5);      /* header: predictor dimension (R18) */
  /* eb_abs exactly as the 1D path (Eq 1, R3) */
  float eb_abs;
  if (mode == 0) {
    if (!eb_usable(eb)) return ORACLE_EINVAL;
    eb_abs = eb;
  } else if (mode == 1) {
    if (!(eb > 0.0f) || !std::isfinite(eb)) return ORACLE_EINVAL;
    float mn, mx;
    oracle_value_range(x, size_t(n), &mn, &mx);
    eb_abs = eb * (mx - mn);
  } else {
    return ORACLE_EINVAL;
  }
  std::memset(out, 0, size_t(HEADER_BYTES + align16(nb)));
  if (!eb_usable(eb_abs)) {                             /* R5 */
    write_header(out, n, mode_byte, ORACLE_ERANGE, eb_abs, eb, 0, L);
    *out_bytes = HEADER_BYTES + align16(nb);
    return ORACLE_ERANGE;
  }
  /* (1) pre-quantisation of every point, the guard of R18 */
  std::vector<int32_t> r(static_cast<size_t>(n));
  if (prequantize_guarded(x, size_t(n), eb_abs, r.data(), dims == 2 ? GUARD2 : GUARD2 / 2) != ORACLE_OK) {
    write_header(out, n, mode_byte, ORACLE_ERANGE, eb_abs, eb, 0, L);
    *out_bytes = HEADER_BYTES + align16(nb);
    return ORACLE_ERANGE;
  }
  /* (1') blocks of the field in raster order, zero outside the field, then
   *      the block-local multi-dimensional Lorenzo prediction */
  int bz, by, bx;
  md_box(dims, &bz, &by, &bx);
  const uint64_t nbz = ceil_div(nz, bz), nby = ceil_div(ny, by), nbx = ceil_div(nx, bx);
  std::vector<int32_t> l(static_cast<size_t>(nb * L));
  uint64_t k = 0;
  for (uint64_t kz = 0; kz < nbz; ++kz)
    for (uint64_t ky = 0; ky < nby; ++ky)
      for (uint64_t kx = 0; kx < nbx; ++kx, ++k) {
        int32_t rb[32];
        for (int z = 0; z < bz; ++z)
          for (int y = 0; y < by; ++y)
            for (int xx = 0; xx < bx; ++xx) {
              const uint64_t gz = kz * bz + z, gy = ky * by + y, gx = kx * bx + xx;
              rb[(z * by + y) * bx + xx] =
                  (gz < nz && gy < ny && gx < nx) ? r[size_t((gz * ny + gy) * nx + gx)] : 0;
            }
        oracle_block_lorenzo_md(rb, dims, &l[size_t(k * L)]);
      }
  /* (2)-(4) exactly as the 1D path */
  const uint64_t payload_bytes = encode_and_place(l.data(), nb, L, out);
  write_header(out, n, mode_byte, ORACLE_OK, eb_abs, eb, payload_bytes, L);
  *out_bytes = HEADER_BYTES + align16(nb) + payload_bytes;
  return ORACLE_OK;
}

int oracle_decompress_md(const uint8_t* in, uint64_t in_bytes, float* out, uint64_t nz,
                         uint64_t ny, uint64_t nx, int dims) {
  if (in == nullptr || out == nullptr || !md_args_ok(nz, ny, nx, dims)) return ORACLE_EINVAL;
  if (in_bytes < uint64_t(HEADER_BYTES)) return ORACLE_ECORRUPT;
  if (!(in[0] == 'C' && in[1] == 'S' && in[2] == 'Z' && in[3] == 'P') || in[4] != 1 || in[7] != 5 ||
      ((in[5] >> 5) & 3) != dims - 1 || (in[5] & 0x10))
    return ORACLE_ECORRUPT;
  if (in[6] != ORACLE_OK) return in[6] == ORACLE_ERANGE ? ORACLE_ERANGE : ORACLE_ECORRUPT;
  const uint64_t n = nz * ny * nx;
  if (get_u64(in + 8) != n) return ORACLE_EINVAL;
  const float eb_abs = get_f32(in + 16);
  const uint64_t payload_bytes = get_u64(in + 24);
  const uint64_t nb = oracle_num_blocks_md(nz, ny, nx, dims);
  const uint64_t p0 = HEADER_BYTES + align16(nb);
  if (in_bytes < p0 || !eb_usable(eb_abs)) return ORACLE_ECORRUPT;
  /* F -> CmpL (Eq 2) -> offsets (Eq 3), as the 1D path */
  const uint8_t* fixed_length = in + HEADER_BYTES;
  std::vector<uint64_t> block_offset(static_cast<size_t>(nb)), sync_offset(static_cast<size_t>(nb));
  for (uint64_t k = 0; k < nb; ++k) {
    if (fixed_length[k] > MAX_F) return ORACLE_ECORRUPT;
    block_offset[k] = oracle_block_bytes(fixed_length[k], L);
  }
  oracle_exclusive_scan(block_offset.data(), size_t(nb), sync_offset.data());
  if (sync_offset[nb - 1] + block_offset[nb - 1] != payload_bytes || in_bytes < p0 + payload_bytes)
    return ORACLE_ECORRUPT;
  int bz, by, bx;
  md_box(dims, &bz, &by, &bx);
  const uint64_t nbz = ceil_div(nz, bz), nby = ceil_div(ny, by), nbx = ceil_div(nx, bx);
  const float two_eb = eb_abs + eb_abs;
  uint64_t k = 0;
  for (uint64_t kz = 0; kz < nbz; ++kz)
    for (uint64_t ky = 0; ky < nby; ++ky)
      for (uint64_t kx = 0; kx < nbx; ++kx, ++k) {
        int32_t l[32], r[32];
        oracle_decode_block_L(in + p0 + sync_offset[k], fixed_length[k], L, l);
        /* inverse prediction, in the block's raster order: r = l + pred(r),
         * the predictor's neighbours all precede the point */
        for (int z = 0; z < bz; ++z)
          for (int y = 0; y < by; ++y)
            for (int xx = 0; xx < bx; ++xx) {
              auto at = [&](int zz, int yy, int x2) -> int32_t {
                if (zz < 0 || yy < 0 || x2 < 0) return 0;
                return r[(zz * by + yy) * bx + x2];
              };
              int32_t pred;
              if (dims == 2)
                pred = at(z, y, xx - 1) + at(z, y - 1, xx) - at(z, y - 1, xx - 1);
              else
                pred = at(z, y, xx - 1) + at(z, y - 1, xx) + at(z - 1, y, xx)
                       - at(z, y - 1, xx - 1) - at(z - 1, y, xx - 1) - at(z - 1, y - 1, xx)
                       + at(z - 1, y - 1, xx - 1);
              r[(z * by + y) * bx + xx] = l[(z * by + y) * bx + xx] + pred;
            }
        /* d' = r * 2eb at the points inside the field */
        for (int z = 0; z < bz; ++z)
          for (int y = 0; y < by; ++y)
            for (int xx = 0; xx < bx; ++xx) {
              const uint64_t gz = kz * bz + z, gy = ky * by + y, gx = kx * bx + xx;
              if (gz < nz && gy < ny && gx < nx)
                out[size_t((gz * ny + gy) * nx + gx)] = float(r[(z * by + y) * bx + xx]) * two_eb;
            }
      }
  return ORACLE_OK;
}

/* Reconstruction quality, each statistic written out by its definition
 * (DESIGN.md sec 9.2): the printed artifact values of P:1918-1933 satisfy
 * exactly these relations (tests/test_oracle_quality.py pins them). */
void oracle_quality(const float* x, const float* y, uint64_t n, double bound, double out[12],
                    uint64_t out_counts[2]) {
  /* value range of the original (Min, Max, range) */
  double mn = x[0], mx = x[0];
  for (uint64_t i = 1; i < n; ++i) {
    if (x[i] < mn) mn = x[i];
    if (x[i] > mx) mx = x[i];
  }
  const double range = mx - mn;
  /* pass 1: means of x and y */
  double sum_x = 0.0, sum_y = 0.0;
  for (uint64_t i = 0; i < n; ++i) {
    sum_x += double(x[i]);
    sum_y += double(y[i]);
  }
  const double mean_x = sum_x / double(n), mean_y = sum_y / double(n);
  /* pass 2: errors and centred sums */
  double max_abs = 0.0, max_pw = 0.0, sum_e2 = 0.0, sum_x2 = 0.0;
  double cxx = 0.0, cyy = 0.0, cxy = 0.0;
  uint64_t over = 0;
  for (uint64_t i = 0; i < n; ++i) {
    const double e = double(x[i]) - double(y[i]);
    const double ae = e < 0 ? -e : e;
    if (ae > max_abs) max_abs = ae;                        /* Max absolute error */
    if (x[i] != 0.0f) {                                    /* Max pw relative error */
      const double ax = x[i] < 0 ? -double(x[i]) : double(x[i]);
      if (ae / ax > max_pw) max_pw = ae / ax;
    }
    if (ae > bound) ++over;
    sum_e2 += e * e;
    sum_x2 += double(x[i]) * double(x[i]);
    const double dx = double(x[i]) - mean_x, dy = double(y[i]) - mean_y;
    cxx += dx * dx;
    cyy += dy * dy;
    cxy += dx * dy;
  }
  const double mse = sum_e2 / double(n);
  out[0] = mn;
  out[1] = mx;
  out[2] = range;
  out[3] = max_abs;
  out[4] = max_abs / range;                                /* Max relative error */
  out[5] = max_pw;
  out[6] = mse;
  out[7] = 20.0 * std::log10(range) - 10.0 * std::log10(mse);   /* PSNR (dB) */
  out[8] = std::sqrt(mse) / range;                         /* NRMSE */
  out[9] = std::sqrt(sum_e2);                              /* normErr */
  out[10] = std::sqrt(sum_e2) / std::sqrt(sum_x2);         /* normErr_norm */
  out[11] = cxy / std::sqrt(cxx * cyy);                    /* pearson coeff */
  out_counts[0] = n;
  out_counts[1] = over;
}

}  // extern "C"
