// linkbench.cu — host-link / HBM micro-benchmarks for the roofline denominators.
//
// MEASURED_PEAKS.json has no host-link figure, so the library measures the two
// routes the hot path uses to reach host memory:
//   * DMA: one cudaMemcpyAsync H2D from pinned memory (step ③);
//   * zero-copy: a streaming-read kernel of coalesced 16-byte loads from a
//     mapped pinned buffer (the kernels' miss path);
// plus an HBM copy kernel (read+write bytes, as MEASURED_PEAKS' hbm_gbs).
#include <cuda_runtime.h>

#include <algorithm>

#include "gcsm.h"

namespace {

__global__ void k_stream_read(const int4 *__restrict__ src, size_t n16, unsigned long long *sink) {
  int4 acc = make_int4(0, 0, 0, 0);
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 3 * stride < n16; i += 4 * stride) {
    const int4 a = src[i], b = src[i + stride], c = src[i + 2 * stride], d = src[i + 3 * stride];
    acc.x ^= a.x ^ b.x ^ c.x ^ d.x;
    acc.y ^= a.y ^ b.y ^ c.y ^ d.y;
    acc.z ^= a.z ^ b.z ^ c.z ^ d.z;
    acc.w ^= a.w ^ b.w ^ c.w ^ d.w;
  }
  for (; i < n16; i += stride) {
    const int4 a = src[i];
    acc.x ^= a.x; acc.y ^= a.y; acc.z ^= a.z; acc.w ^= a.w;
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345678) atomicAdd(sink, 1ull);
}

__global__ void k_copy(const int4 *__restrict__ src, int4 *__restrict__ dst, size_t n16) {
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride) dst[i] = src[i];
}

}  // namespace

extern "C" gcsm_status gcsm_measure_host_link(int32_t device, uint64_t bytes, double *zero_copy_gbps,
                                              double *dma_h2d_gbps, double *hbm_copy_gbps) {
  if (bytes < (1u << 20)) return GCSM_EINVAL;
  bytes &= ~uint64_t(15);
  if (device >= 0 && cudaSetDevice(device) != cudaSuccess) return GCSM_EDEVICE;
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  void *h = nullptr, *hd = nullptr, *d = nullptr, *d2 = nullptr;
  unsigned long long *sink = nullptr;
  cudaStream_t s = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  gcsm_status st = GCSM_OK;
  float best_zc = 1e30f, best_dma = 1e30f, best_cp = 1e30f;
  if (cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess ||
      cudaHostGetDevicePointer(&hd, h, 0) != cudaSuccess || cudaMalloc(&d, bytes) != cudaSuccess ||
      cudaMalloc(&d2, bytes) != cudaSuccess || cudaMalloc(&sink, 8) != cudaSuccess ||
      cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess || cudaEventCreate(&e0) != cudaSuccess ||
      cudaEventCreate(&e1) != cudaSuccess) {
    st = GCSM_ENOMEM;
    goto done;
  }
  for (size_t i = 0; i < bytes / 4; i += 1024) ((int *)h)[i] = (int)i;
  for (int rep = 0; rep < 6; ++rep) {
    float ms = 0;
    cudaEventRecord(e0, s);
    cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice, s);
    cudaEventRecord(e1, s);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    if (rep) best_dma = std::min(best_dma, ms);
    cudaEventRecord(e0, s);
    k_stream_read<<<sms * 8, 256, 0, s>>>((const int4 *)hd, bytes / 16, sink);
    cudaEventRecord(e1, s);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    if (rep) best_zc = std::min(best_zc, ms);
    cudaEventRecord(e0, s);
    k_copy<<<sms * 8, 256, 0, s>>>((const int4 *)d, (int4 *)d2, bytes / 16);
    cudaEventRecord(e1, s);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    if (rep) best_cp = std::min(best_cp, ms);
  }
  if (cudaGetLastError() != cudaSuccess) {
    st = GCSM_EDEVICE;
    goto done;
  }
  if (zero_copy_gbps) *zero_copy_gbps = (double)bytes / (best_zc * 1e-3) / 1e9;
  if (dma_h2d_gbps) *dma_h2d_gbps = (double)bytes / (best_dma * 1e-3) / 1e9;
  if (hbm_copy_gbps) *hbm_copy_gbps = 2.0 * (double)bytes / (best_cp * 1e-3) / 1e9;
done:
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  if (s) cudaStreamDestroy(s);
  if (sink) cudaFree(sink);
  if (d2) cudaFree(d2);
  if (d) cudaFree(d);
  if (h) cudaFreeHost(h);
  return st;
}
