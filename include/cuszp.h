/*
 * cuszp.h -- C ABI of the B200-native (sm_100a) cuSZp hot path.
 *
 * Method: Huang et al., "cuSZp: An Ultra-fast GPU Error-bounded Lossy
 * Compression Framework with Optimized End-to-End Performance", SC'23.
 * "P:NNN" cites line NNN of the paper text.  Readings of the
 * paper (R1..R16) and the byte format are in DESIGN.md sections 3 and 4.
 *
 * Library: paper_conf_sc_huangd0lc23_b200/libcuszp.so (CUDA runtime linked
 * statically).  Every symbol below is extern "C"; there are no C++ or torch
 * types in any signature.  `stream` is a cudaStream_t passed as void*
 * (NULL = legacy default stream).
 *
 * Conventions shared by all calls
 * -------------------------------
 *  - d_ pointers are CUDA device pointers, h_ pointers host pointers.
 *  - The caller owns (allocates, frees) every buffer.  The asynchronous
 *    calls never allocate, never synchronise and are CUDA-Graph capturable.
 *  - Device buffers must be 16-byte aligned (d_in of cuszp_range: 4-byte).
 *  - A workspace d_ws of cuszp_workspace_bytes(n) bytes must be ZEROED ONCE
 *    when allocated (e.g. cudaMemset) and may then be reused for any number
 *    of calls with element counts <= n.  Calls sharing a workspace must be
 *    ordered (same stream, or event-ordered); concurrent calls need distinct
 *    workspaces.
 *  - Return value: CUSZP_OK, or a SYNCHRONOUS error detected on the host
 *    (bad argument, too-small buffer, CUDA launch failure) -- nothing is
 *    launched in that case.  DATA-DEPENDENT errors are ASYNCHRONOUS: they
 *    are written to the stream header's status byte (compress) and to the
 *    workspace; read them with cuszp_last_status() (synchronising).
 */
#ifndef CUSZP_H
#define CUSZP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CUSZP_BLOCK_LEN 32      /* L, R1: pinned by Table 3's max CR 127.99 */
#define CUSZP_HEADER_BYTES 32   /* R10 */
#define CUSZP_VERSION 1

typedef enum { CUSZP_ABS = 0, CUSZP_REL = 1 } cuszp_mode;

typedef enum {
  CUSZP_OK = 0,
  CUSZP_EINVAL = 1,    /* bad argument (sync) / n != header n (async, decompress) */
  CUSZP_ECUDA = 2,     /* CUDA error while launching or copying (sync) */
  CUSZP_ERANGE = 3,    /* async: |d/2eb| >= 2^22, NaN/Inf data, unusable REL eb (R5) */
  CUSZP_ECORRUPT = 4,  /* async: malformed stream (magic, F > 24, sizes, bounds) */
  CUSZP_ENOSPACE = 5   /* sync: output or workspace too small */
} cuszp_status;

/* The 32-byte stream header, little-endian. */
typedef struct {
  char magic[4];           /* "CSZP" */
  uint8_t version;         /* CUSZP_VERSION */
  uint8_t mode;            /* cuszp_mode */
  uint8_t status;          /* cuszp_status of the compression */
  uint8_t log2_block_len;  /* 5 */
  uint64_t n;              /* number of fp32 elements */
  float eb_abs;            /* absolute bound used: delta (ABS) or lambda*(max-min) (REL, Eq 1) */
  float eb_in;             /* user bound: delta (ABS) or lambda (REL) */
  uint64_t payload_bytes;  /* sum of CmpL_k (Eq 2, Eq 3 total) */
} cuszp_header;

/* Output buffer size for n elements: 32 + align16(nb) + 128*nb, nb =
 * ceil(n/32).  A valid stream is at most 32 + align16(nb) + 100*nb (F <= 24
 * by the R5 guard, CmpL <= 4*25); data that fail the guard are only known to
 * be ERANGE at the end of the kernel and may have written up to 32 words per
 * block by then.  Output buffers of compress must be at least this large. */
size_t cuszp_max_compressed_bytes(size_t n);

/* Exact compressed size from the per-block fixed lengths F[0..nb) (host
 * helper of Eq 2 + Eq 3): 32 + align16(nb) + sum_{F>0} 4(F+1). */
size_t cuszp_compressed_bytes_from_F(const uint8_t* h_F, size_t nb);

/* Workspace bytes for calls with up to n elements (look-back status words,
 * tile ticket, range accumulators). */
size_t cuszp_workspace_bytes(size_t n);

/* a1 -- value range (Eq 1; R3, R4).  One kernel: 128-bit loads,
 * warp/CTA reductions, one atomic per CTA on order-preserving integer keys;
 * the last CTA writes (min, max) to d_minmax[0..1] (NaN if any NaN) and to
 * the workspace.  d_minmax may be NULL.  n must be > 0. */
int cuszp_range(const float* d_in, size_t n, float* d_minmax,
                void* d_ws, size_t ws_bytes, void* stream);

/* a1..a8 -- compression (sec 3.1, Fig 2; sec 4).  mode ABS: eb = delta;
 * mode REL: eb = lambda and eb_abs = lambda*(max-min) is computed ON THE
 * DEVICE (range kernel, then the fused compression kernel -- 2 launches;
 * ABS: 1 launch).  Writes the stream to d_out and its
 * exact length to *d_out_bytes (device u64, may be NULL).
 * Sync errors: EINVAL (NULL pointers with n > 0, mode, eb <= 0 or
 * non-finite, ABS eb not a normal float), ENOSPACE (out_capacity <
 * cuszp_max_compressed_bytes(n), ws_bytes < cuszp_workspace_bytes(n)),
 * ECUDA.  Async: ERANGE in the header status byte and the workspace. */
int cuszp_compress(const float* d_in, size_t n, float eb, int mode,
                   void* d_out, size_t out_capacity,
                   unsigned long long* d_out_bytes,
                   void* d_ws, size_t ws_bytes, void* stream);

/* REL compression of one shard against a GLOBAL value range given on the
 * device as n_pairs (min, max) float pairs (the sharded driver's NCCL
 * all-gather result).  eb_abs = lambda*(max_p max -
 * min_p min).  One launch. */
int cuszp_compress_minmax(const float* d_in, size_t n, float lambda,
                          const float* d_minmax, int n_pairs,
                          void* d_out, size_t out_capacity,
                          unsigned long long* d_out_bytes,
                          void* d_ws, size_t ws_bytes, void* stream);

/* a9..a12 -- decompression (sec 3.2, Fig 3): one fused kernel.  Reads the
 * header on the device; n must equal the header's n (else async EINVAL).
 * in_bytes bounds every read (corrupt offsets -> async ECORRUPT, nothing
 * is read past d_in + in_bytes).  Writes d_out[0..n). */
int cuszp_decompress(const void* d_in, size_t in_bytes, float* d_out, size_t n,
                     void* d_ws, size_t ws_bytes, void* stream);

/* ---- block-length variants L in {8, 16, 32, 64, 128}
 * (the lengths of the paper's smoothness analysis).  Eq 2 is
 * CmpL = (F+1) L/8 bytes; a plane is L/8 bytes with element j at byte j/8,
 * bit j%8 (R9 generalised); header byte 7 = log2(L); one F byte
 * per L-block.  The calls without _L are the L = 32 ones.  Output buffers
 * need cuszp_max_compressed_bytes_L(n, L) bytes (32 + align16(nb) +
 * 32 L/8 nb, nb = ceil(n/L)); workspaces are sized as for L = 32.
 * block_len outside {8, 16, 32, 64, 128}: EINVAL (the size helper returns 0).
 * L = 8 / 16 run the same one-pass kernels with byte-granular placement
 * (a plane is 1 / 2 bytes; one block per lane); same statuses.
 * Decompression must be given the stream's L (a header with another L:
 * async ECORRUPT). */
size_t cuszp_max_compressed_bytes_L(size_t n, int block_len);
int cuszp_compress_L(const float* d_in, size_t n, float eb, int mode, int block_len,
                     void* d_out, size_t out_capacity, unsigned long long* d_out_bytes,
                     void* d_ws, size_t ws_bytes, void* stream);
int cuszp_compress_minmax_L(const float* d_in, size_t n, float lambda,
                            const float* d_minmax, int n_pairs, int block_len,
                            void* d_out, size_t out_capacity, unsigned long long* d_out_bytes,
                            void* d_ws, size_t ws_bytes, void* stream);
int cuszp_decompress_L(const void* d_in, size_t in_bytes, float* d_out, size_t n, int block_len,
                       void* d_ws, size_t ws_bytes, void* stream);

/* ---- 2-layer Lorenzo predictor ----
 * order 1: the paper's 1D 1-layer predictor (the calls above); order 2:
 * l_i = r_i - 2 r_{i-1} + r_{i-2} inside each block (r_{-1} = r_{-2} = 0),
 * R5 guard |r0| < 2^21 (so F <= 24), header mode byte bit 4 (0x10) set;
 * block_len must be 32 for order 2.  Decompression must be given the
 * stream's order (another order in the header: async ECORRUPT).  Sizes and
 * errors as for the _L calls; order outside {1, 2}: EINVAL. */
int cuszp_compress_ex(const float* d_in, size_t n, float eb, int mode, int block_len, int order,
                      void* d_out, size_t out_capacity, unsigned long long* d_out_bytes,
                      void* d_ws, size_t ws_bytes, void* stream);
int cuszp_decompress_ex(const void* d_in, size_t in_bytes, float* d_out, size_t n, int block_len,
                        int order, void* d_ws, size_t ws_bytes, void* stream);

/* Status of the last compress/decompress call made with this workspace.
 * SYNCHRONISES `stream`.  Returns a cuszp_status (or ECUDA). */
int cuszp_last_status(const void* d_ws, void* stream);

/* Copies the 32-byte header of a device stream to *h_hdr.  Synchronises. */
int cuszp_read_header(const void* d_stream, cuszp_header* h_hdr, void* stream);

/* End-to-end calls on HOST buffers (the e2e metric): H2D copy of the input,
 * the device call, D2H of the result; synchronises before returning.
 * Scratch device buffers are caller-owned (sizes as for the device calls);
 * pinned host buffers give asynchronous copies.
 * compress: h_out receives the stream, *h_out_bytes its exact length. */
int cuszp_compress_host(const float* h_in, size_t n, float eb, int mode,
                        void* h_out, size_t out_capacity, size_t* h_out_bytes,
                        float* d_in_scratch, void* d_out_scratch,
                        void* d_ws, size_t ws_bytes, void* stream);
int cuszp_decompress_host(const void* h_in, size_t in_bytes, float* h_out, size_t n,
                          void* d_in_scratch, float* d_out_scratch,
                          void* d_ws, size_t ws_bytes, void* stream);

/* Fully ASYNCHRONOUS host-buffer calls (stream-ordered, no host sync), so
 * consecutive calls on different streams overlap both directions of the
 * host link.  h_in of compress and h_out of decompress: pinned host memory
 * (bulk copies on the copy engines).  h_out / h_out_bytes of compress and
 * h_in of decompress: pinned AND device-mapped host memory (cudaHostAlloc;
 * any pinned allocation under unified addressing): the compressed stream,
 * whose length only the device knows, is moved by an SM copy kernel that
 * reads that length on the device -- exactly the stream's bytes cross the
 * link.  compress: out_capacity >= cuszp_max_compressed_bytes(n) (else
 * ENOSPACE); *h_out_bytes receives the stream length when the stream
 * completes.  decompress: the stream's length is taken from its own header
 * (at most in_capacity bytes are read; d_in_scratch holds in_capacity).
 * Alignment: h_out, h_in (mapped sides) and both device scratch buffers
 * 16-byte aligned, h_out_bytes 8-byte aligned (the copy kernels move 16-
 * and 8-byte words); checked before anything is launched.
 * Sync errors: EINVAL (NULL, unmapped or misaligned buffers), ENOSPACE,
 * ECUDA -- on a sync error nothing has been launched; data errors are
 * asynchronous as for the device calls.  One workspace per stream. */
int cuszp_compress_host_async(const float* h_in, size_t n, float eb, int mode,
                              void* h_out, size_t out_capacity, unsigned long long* h_out_bytes,
                              float* d_in_scratch, void* d_out_scratch,
                              void* d_ws, size_t ws_bytes, void* stream);
int cuszp_decompress_host_async(const void* h_in, size_t in_capacity, float* h_out, size_t n,
                                void* d_in_scratch, float* d_out_scratch,
                                void* d_ws, size_t ws_bytes, void* stream);

/* ---- multi-dimensional Lorenzo ----
 * "Lorenzo predictions with higher dimensions" inside blocks (DESIGN R18).
 * The field is an (nz, ny, nx) array, x fastest, n = nz*ny*nx (nz = 1 for a
 * 2D field).  dims = 2: an L = 32 block is a 1 x 4 x 8 box of the field,
 * dims = 3: a 2 x 4 x 4 box; blocks tile the field in raster order of the
 * block grid (x fastest), points outside the field are quantisation
 * integer 0 (R8), and the block-local predictor takes neighbours outside
 * the block as 0:  dims 2: l = r - r(x-1) - r(y-1) + r(y-1,x-1);  dims 3:
 * the 7-term Lorenzo predictor.  Guard |round(d/2eb)| < 2^21 (dims 2) or
 * 2^20 (dims 3), else ERANGE.  Stream: the L = 32 format with nb =
 * cuszp_num_blocks_md() blocks; header mode byte bits 5-6 = dims - 1.  The
 * shape is not stored: decompression takes it (like n).  Buffers: output
 * cuszp_max_compressed_bytes_md, workspace cuszp_workspace_bytes_md (zeroed
 * once, like every workspace).  Sync errors: EINVAL (dims not 2 or 3, a zero
 * extent, > 2^32 blocks, NULL / misaligned pointers, eb as for
 * cuszp_compress), ENOSPACE, ECUDA; data errors asynchronous as usual. */
size_t cuszp_num_blocks_md(size_t nz, size_t ny, size_t nx, int dims);
size_t cuszp_max_compressed_bytes_md(size_t nz, size_t ny, size_t nx, int dims);
size_t cuszp_workspace_bytes_md(size_t nz, size_t ny, size_t nx, int dims);
int cuszp_compress_md(const float* d_in, size_t nz, size_t ny, size_t nx, int dims, float eb, int mode,
                      void* d_out, size_t out_capacity, unsigned long long* d_out_bytes,
                      void* d_ws, size_t ws_bytes, void* stream);
int cuszp_decompress_md(const void* d_in, size_t in_bytes, float* d_out, size_t nz, size_t ny, size_t nx,
                        int dims, void* d_ws, size_t ws_bytes, void* stream);

/* ---- reconstruction quality on the device ----
 * The statistics the paper's artifact reads off QCAT compareData
 * (P:1918-1933), PSNR as in sec 2.1, all in fp64.  x = original,
 * y = reconstruction, e_i = x_i - y_i (exact in fp64):
 *   min, max, range = max - min of x;
 *   max_abs_err = max |e_i|;  max_rel_err = max_abs_err / range;
 *   max_pw_rel_err = max over x_i != 0 of |e_i| / |x_i|;
 *   mse = sum e_i^2 / n;  psnr = 20 log10(range) - 10 log10(mse);
 *   nrmse = sqrt(mse) / range;  norm_err = sqrt(sum e_i^2);
 *   norm_err_norm = norm_err / sqrt(sum x_i^2);
 *   pearson = sum (x-mx)(y-my) / sqrt(sum (x-mx)^2 sum (y-my)^2);
 *   n_over_bound = #{i : |e_i| > bound}  (pass the eb_abs of the stream).
 * Degenerate inputs follow IEEE (range 0 -> inf/NaN ratios; mse 0 -> psnr
 * +inf).  Inputs are expected finite. */
typedef struct cuszp_quality_stats {
  double min, max, range;
  double max_abs_err, max_rel_err, max_pw_rel_err;
  double mse, psnr, nrmse;
  double norm_err, norm_err_norm, pearson;
  unsigned long long n, n_over_bound;
} cuszp_quality_stats;

/* Workspace of cuszp_quality (independent of n); caller-zeroed once,
 * left zeroed by every call. */
size_t cuszp_quality_workspace_bytes(void);

/* One kernel, one pass over d_x and d_y (8n bytes), writes *d_q (device
 * memory, 8-byte aligned) stream-ordered.  Sums are folded in a fixed
 * order: the result is deterministic for a given device.
 * Sync errors: EINVAL (NULL pointers, n = 0, misaligned pointers, NaN
 * bound), ENOSPACE (ws_bytes too small), ECUDA. */
int cuszp_quality(const float* d_x, const float* d_y, size_t n, double bound,
                  cuszp_quality_stats* d_q, void* d_ws, size_t ws_bytes, void* stream);

/* ---- sharded container, one-sided gather ----------
 * Container v2: u64 words magic "CSZPCONT", version 2,
 * P, n_total, n_p[P], bytes_p[P], offset_p[P] (offsets of the 16-byte
 * aligned shards, relative to the header's end), the header padded to 16
 * bytes.  cuszp_container_put copies shard p (d_shard, this rank's stream,
 * 16-byte aligned) into the container at d_container (any device address
 * the calling GPU can write: its own memory or a peer GPU's, mapped by CUDA
 * IPC / UVA; 16-byte aligned) at the offset d_header (the container header
 * words, device memory, 8-byte aligned) gives it -- read ON THE DEVICE, so a
 * gather needs no host round trip -- followed by zeros up to align16(bytes_p)
 * (so d_container needs room for the padded shard); with write_header != 0
 * it also writes the header words and their zero padding.  The caller orders the puts of
 * all ranks before the container is read (e.g. an NCCL all-reduce after the
 * put on every rank's stream).  Sync errors: EINVAL (NULL pointers, P = 0,
 * p >= P, misalignment), ECUDA; the copy itself has no data-dependent
 * errors (bytes_p and offset_p are trusted: they come from the all-gather
 * of the compressed sizes). */
int cuszp_container_put(const void* d_shard, const void* d_header, unsigned P, unsigned p, void* d_container,
                        int write_header, void* stream);

/* Human-readable status name. */
const char* cuszp_status_string(int status);

/* CUSZP_VERSION * 100 + build id. */
int cuszp_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CUSZP_H */
