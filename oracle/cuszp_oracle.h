/*
 * cuszp_oracle.h -- plain, slow, single-threaded CPU oracle of cuSZp
 * (Huang et al., SC'23, "cuSZp: An Ultra-fast GPU Error-bounded Lossy
 * Compression Framework with Optimized End-to-End Performance").
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product path (paper_conf_sc_huangd0lc23_b200/) never links, imports
 * or calls anything in oracle/, and this file shares no code, header,
 * table or constant generator with the CUDA path.
 *
 * Citations: "P:NNN" = line NNN of the paper text with the
 * section / equation / figure it falls in.  Readings of ambiguous passages
 * are the ones listed in DESIGN.md section 3 ("Readings of the paper").
 *
 * Parity status: every function below is pinned by tests/test_oracle_*.py
 * (golden blocks, closed forms, exact-arithmetic brute force, invariants);
 * the only unpinned item is byte compatibility with the original, never
 * released cuSZp binary ("parity unpinned" for that comparison).
 */
#ifndef CUSZP_ORACLE_H
#define CUSZP_ORACLE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Status codes (same numeric meaning as the product ABI; written out
 * independently here). */
enum {
  ORACLE_OK = 0,
  ORACLE_EINVAL = 1,
  ORACLE_ERANGE = 3,
  ORACLE_ECORRUPT = 4,
  ORACLE_ENOSPACE = 5
};

/* ---- individual steps of the method (each pinned on its own) ---------- */

/* Eq 1 (sec 2.1): eb_abs = delta (ABS) or lambda * (max - min)
 * (REL).  Writes exact min and max of x[0..n).  n must be > 0. */
void oracle_value_range(const float* x, size_t n, float* mn, float* mx);

/* Pre-quantisation r_i = round(d_i / 2eb) (sec 4.1).
 * Writes q[0..n).  Returns ORACLE_OK or ORACLE_ERANGE (guard, DESIGN R5). */
int oracle_prequantize(const float* x, size_t n, float eb_abs, int32_t* q);

/* 1D 1-layer Lorenzo inside each L=32 block (sec 4.1):
 * l_i = r_i - r_{i-1}, r_{-1} := 0 at every block start.  q and l have
 * nb*32 entries (caller pads q with zeros past n, DESIGN R8). */
void oracle_block_lorenzo(const int32_t* q, size_t nb, int32_t* l);

/* "position of the last non-zero bit" of m (sec 4.2). */
int oracle_bit_length(uint32_t m);

/* Eq 2: CmpL = (F+1) * L / 8 bytes for a non-zero block,
 * 0 for a zero block (DESIGN R6). */
uint64_t oracle_block_bytes(int F, int L);

/* Eq 3: exclusive prefix sum of the block offset array. */
void oracle_exclusive_scan(const uint64_t* cmpl, size_t k, uint64_t* sync_off);

/* Fixed-length encoding + block bit-shuffle of ONE block of 32 Lorenzo
 * integers (sec 4.2, sec 4.4).  Returns F and writes
 * CmpL = oracle_block_bytes(F, 32) payload bytes to out. */
int oracle_encode_block(const int32_t l[32], uint8_t* out);

/* Inverse of oracle_encode_block (sec 3.2). */
void oracle_decode_block(const uint8_t* payload, int F, int32_t l[32]);

/* ---- the whole path ---------------------------------------------------- */

/* Largest stream for n elements: 32 + align16(nb) + 100 * nb. */
uint64_t oracle_max_compressed_bytes(uint64_t n);

/* Compress (sec 3.1, Fig 2).  mode 0 = ABS (eb is delta), 1 = REL (eb is
 * lambda).  Writes the stream to out (capacity cap) and its length to
 * *out_bytes.  Returns a status; on ORACLE_ERANGE the stream header carries
 * status 3 and the payload is not meaningful. */
int oracle_compress(const float* x, uint64_t n, float eb, int mode,
                    uint8_t* out, uint64_t cap, uint64_t* out_bytes);

/* REL compression of one shard against a global value range given as
 * n_pairs (min, max) pairs (the sharded driver's contract). */
int oracle_compress_minmax(const float* x, uint64_t n, float lambda,
                           const float* minmax, int n_pairs,
                           uint8_t* out, uint64_t cap, uint64_t* out_bytes);

/* Decompress (sec 3.2, Fig 3).  n must equal the header's n. */
int oracle_decompress(const uint8_t* in, uint64_t in_bytes, float* out,
                      uint64_t n);

/* ---- block-length variants ---------------------
 * The same method with block length L in {8, 16, 32, 64, 128} (the lengths
 * of the paper's smoothness analysis; Eq 2 is CmpL = (F+1) L/8
 * bytes, the bit-shuffle puts bit k of every |l_j| into the k-th group of
 * L/8 bytes).  Header byte 7 = log2(L); oracle_decompress reads
 * it.  The functions without _L are the L = 32 ones. */
void oracle_block_lorenzo_L(const int32_t* q, size_t nb, int L, int32_t* l);
int oracle_encode_block_L(const int32_t* l, int L, uint8_t* out);
void oracle_decode_block_L(const uint8_t* payload, int F, int L, int32_t* l);
uint64_t oracle_max_compressed_bytes_L(uint64_t n, int L);
int oracle_compress_L(const float* x, uint64_t n, float eb, int mode, int L,
                      uint8_t* out, uint64_t cap, uint64_t* out_bytes);
int oracle_compress_minmax_L(const float* x, uint64_t n, float lambda,
                             const float* minmax, int n_pairs, int L,
                             uint8_t* out, uint64_t cap, uint64_t* out_bytes);

/* ---- 2-layer Lorenzo (DESIGN R17) --
 * order 2: l_i = r_i - 2 r_{i-1} + r_{i-2} inside each block (r_{-1} =
 * r_{-2} = 0), guard |r0| < 2^21 so F <= 24; header mode byte bit 4 (0x10)
 * marks it and oracle_decompress inverts it.  order 1 = oracle_compress_L. */
int oracle_compress_ex(const float* x, uint64_t n, float eb, int mode, int L, int order,
                       uint8_t* out, uint64_t cap, uint64_t* out_bytes);

/* ---- multi-dimensional Lorenzo inside blocks -----
 * "Lorenzo predictions with higher dimensions" (the Lorenzo
 * predictor of ref [14]), DESIGN R18.  The field has shape (nz, ny, nx), x
 * fastest, n = nz*ny*nx.  An L = 32 block is a 1 x 4 x 8 (dims = 2) or
 * 2 x 4 x 4 (dims = 3) box of the field; blocks tile the field in raster
 * order of the block grid (ceil(nz/bz), ceil(ny/4), ceil(nx/bx)), x
 * fastest; element j of a block is (z*4 + y)*bx + x.  Elements outside the
 * field are quantisation integer 0 (R8), and the predictor treats
 * neighbours outside the BLOCK as 0 (block-local, like P:525-529):
 *   dims 2: l = r - r(y,x-1) - r(y-1,x) + r(y-1,x-1)
 *   dims 3: l = r - r(x-1) - r(y-1) - r(z-1) + r(y-1,x-1) + r(z-1,x-1)
 *               + r(z-1,y-1) - r(z-1,y-1,x-1)            (same z/y/x otherwise)
 * Guard |r0| < 2^21 (dims 2) or 2^20 (dims 3) so |l| < 2^23 and F <= 24.
 * Stream: the L = 32 format with nb = the number of grid blocks, header
 * mode byte bits 5-6 = dims - 1; the shape is the caller's (like n).
 * dims = 1 is oracle_compress (the 1D predictor, blocks of 32 in order). */
uint64_t oracle_num_blocks_md(uint64_t nz, uint64_t ny, uint64_t nx, int dims);
uint64_t oracle_max_compressed_bytes_md(uint64_t nz, uint64_t ny, uint64_t nx, int dims);
void oracle_block_lorenzo_md(const int32_t r[32], int dims, int32_t l[32]);
int oracle_compress_md(const float* x, uint64_t nz, uint64_t ny, uint64_t nx, int dims, float eb,
                       int mode, uint8_t* out, uint64_t cap, uint64_t* out_bytes);
int oracle_decompress_md(const uint8_t* in, uint64_t in_bytes, float* out, uint64_t nz,
                         uint64_t ny, uint64_t nx, int dims);

/* ---- reconstruction quality -------------------
 * The statistics of the paper's artifact output (QCAT compareData,
 * P:1918-1933) and PSNR (sec 2.1), in fp64, two plain passes
 * (means first, then centred sums).  out[0..11] = min, max, range,
 * max_abs_err, max_rel_err, max_pw_rel_err, mse, psnr, nrmse, norm_err,
 * norm_err_norm, pearson; out_counts[0..1] = n, #{|x_i - y_i| > bound}.
 * n must be > 0.  Pinned by the artifact's printed values, closed forms and
 * numpy's corrcoef; norm_err_norm (= ||e||_2 / ||x||_2, reading Q2 of
 * DESIGN.md 9.2) by hand-computed closed forms and by the printed triple
 * (normErr, normErr_norm, pearson): the printed Pearson coefficient rules out
 * a centred normalisation, and an input with the printed RMSE and Pearson
 * coefficient reproduces the printed 0.015479 (tests/test_oracle_quality.py). */
void oracle_quality(const float* x, const float* y, uint64_t n, double bound,
                    double out[12], uint64_t out_counts[2]);

#ifdef __cplusplus
}
#endif
#endif /* CUSZP_ORACLE_H */
