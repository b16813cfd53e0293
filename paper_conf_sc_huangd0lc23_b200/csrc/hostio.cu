// hostio.cu -- fully asynchronous host-buffer entry points (the e2e path:
// inputs in pinned host memory, results back in pinned host memory).
//
// The compressed stream's length is only known on the device, so its
// transfers are done by SM copy kernels over PCIe on host-MAPPED pinned
// memory (zero-copy), which read the length on the device: no host
// round trip, no synchronisation, so consecutive calls on different streams
// overlap the host->device and device->host directions of the link.  The
// bulk fp32 transfers (4n bytes each way) stay on the copy engines
// (cudaMemcpyAsync).
#include "internal.cuh"

namespace cuszp {

namespace {

constexpr int kIoThreads = 256;

// dst[0..len) = src[0..len), len = *d_len (device) clamped to cap.
// 16-byte vectors when both ends allow it (our buffers always do).
__global__ void __launch_bounds__(kIoThreads) copy_len_kernel(uint8_t* dst, const uint8_t* src,
                                                              const unsigned long long* d_len, uint64_t cap,
                                                              unsigned long long* len_out) {
  uint64_t len = *d_len;
  if (len > cap) len = cap;
  if (len_out && blockIdx.x == 0 && threadIdx.x == 0) *len_out = len;
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t nth = uint64_t(gridDim.x) * blockDim.x;
  const uint64_t n16 = len / 16;
  uint4* d4 = reinterpret_cast<uint4*>(dst);
  const uint4* s4 = reinterpret_cast<const uint4*>(src);
  uint64_t i = tid;
  for (; i + 3 * nth < n16; i += 4 * nth) {   // 4 independent 16-byte transfers in flight
    const uint4 a = s4[i], b = s4[i + nth], c = s4[i + 2 * nth], d = s4[i + 3 * nth];
    d4[i] = a;
    d4[i + nth] = b;
    d4[i + 2 * nth] = c;
    d4[i + 3 * nth] = d;
  }
  for (; i < n16; i += nth) d4[i] = s4[i];
  for (uint64_t k = n16 * 16 + tid; k < len; k += nth) dst[k] = src[k];
}

// Length of a host-resident stream read from its own header (n = header n,
// checked by the decompression kernel): 32 + align16(nb) + payload_bytes.
__global__ void stream_len_kernel(const uint8_t* h_stream, uint64_t n, unsigned long long* d_len) {
  const uint64_t payload = *reinterpret_cast<const volatile uint64_t*>(h_stream + 24);
  const uint64_t nb = (n + kL - 1) / kL;
  *d_len = (n == 0) ? uint64_t(kHdr) : uint64_t(kHdr) + align16(nb) + payload;
}

// Shard p of a container: bytes_p = hdr[4 + P + p] bytes
// from `shard` to cont + header_bytes(P) + hdr[4 + 2P + p], both 16-byte
// aligned (offsets are align16-padded), then zeros up to align16(bytes_p);
// with write_header also the header words and their zero padding.  `cont` may be a peer GPU's memory (UVA).
__global__ void __launch_bounds__(kIoThreads) container_put_kernel(const uint8_t* shard, const int64_t* hdr,
                                                                   uint32_t P, uint32_t p, uint8_t* cont,
                                                                   int write_header) {
  const uint64_t hw = 4ull + 3ull * P;                       // header words
  const uint64_t base = (8 * hw + 15) / 16 * 16;
  const uint64_t bytes = uint64_t(hdr[4 + P + p]);
  uint8_t* dst = cont + base + uint64_t(hdr[4 + 2ull * P + p]);
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t nth = uint64_t(gridDim.x) * blockDim.x;
  const uint64_t n16 = bytes / 16;
  uint4* d4 = reinterpret_cast<uint4*>(dst);
  const uint4* s4 = reinterpret_cast<const uint4*>(shard);
  uint64_t i = tid;
  for (; i + 3 * nth < n16; i += 4 * nth) {   // 4 independent 16-byte transfers in flight
    const uint4 a = s4[i], b = s4[i + nth], c = s4[i + 2 * nth], d = s4[i + 3 * nth];
    d4[i] = a;
    d4[i + nth] = b;
    d4[i + 2 * nth] = c;
    d4[i + 3 * nth] = d;
  }
  for (; i < n16; i += nth) d4[i] = s4[i];
  for (uint64_t k = n16 * 16 + tid; k < bytes; k += nth) dst[k] = shard[k];
  for (uint64_t k = bytes + tid; k < (bytes + 15) / 16 * 16; k += nth) dst[k] = 0;   // the shard's zero padding
  if (write_header) {
    int64_t* h = reinterpret_cast<int64_t*>(cont);
    for (uint64_t k = tid; k < hw; k += nth) h[k] = hdr[k];
    for (uint64_t k = 8 * hw + tid; k < base; k += nth) cont[k] = 0;
  }
}

}  // namespace

int launch_container_put(const void* shard, const void* hdr, uint32_t P, uint32_t p, void* cont, int write_header,
                         int sms, cudaStream_t s) {
  container_put_kernel<<<unsigned(sms) * 2, kIoThreads, 0, s>>>(static_cast<const uint8_t*>(shard),
                                                                 static_cast<const int64_t*>(hdr), P, p,
                                                                 static_cast<uint8_t*>(cont), write_header);
  return cudaGetLastError() == cudaSuccess ? CUSZP_OK : CUSZP_ECUDA;
}

int launch_copy_len(void* dst, const void* src, const unsigned long long* d_len, uint64_t cap,
                    unsigned long long* len_out, int sms, cudaStream_t s) {
  uint64_t want = (cap / 16 + kIoThreads - 1) / kIoThreads;
  uint64_t grid = uint64_t(sms) * 4;
  if (grid > want) grid = want;
  if (grid < 1) grid = 1;
  copy_len_kernel<<<unsigned(grid), kIoThreads, 0, s>>>(static_cast<uint8_t*>(dst), static_cast<const uint8_t*>(src),
                                                         d_len, cap, len_out);
  return cudaGetLastError() == cudaSuccess ? CUSZP_OK : CUSZP_ECUDA;
}

int launch_stream_len(const void* h_stream_dev, uint64_t n, unsigned long long* d_len, cudaStream_t s) {
  stream_len_kernel<<<1, 1, 0, s>>>(static_cast<const uint8_t*>(h_stream_dev), n, d_len);
  return cudaGetLastError() == cudaSuccess ? CUSZP_OK : CUSZP_ECUDA;
}

}  // namespace cuszp
