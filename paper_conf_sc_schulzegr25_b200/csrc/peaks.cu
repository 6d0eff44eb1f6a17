// peaks.cu — measured instruction-throughput peaks of this GPU (diagnostics, not the hot
// path): the denominators bench.py uses for the kernels whose roofline is a pipe, not HBM or
// the tensor cores: T3 SIMT contractions (fp32 FFMA) and T5 PRL (integer /
// half compares, bound by instruction issue).
//   ffma  — 8 independent FFMA chains per thread (fma pipe), flop = 2 per FFMA
//   alu   — 8 independent LOP3 chains per thread (alu pipe)
//   issue — the best sustained instruction rate (thread-instructions/s): the FFMA kernel's
//           (FFMA issues every cycle; LOP3 is half-rate — measured on B200: 35.8 vs 18.4
//           T thread-instructions/s) or a 4 FFMA + 4 LOP3 interleave, whichever is higher
// Every kernel runs 4 resident CTAs of 256 threads per SM for ~20 ms; the result is the
// best of 3 launches timed with CUDA events.
#include <cuda_runtime.h>

#include <algorithm>

#include "internal.h"

namespace mdh {

constexpr int PK_THREADS = 256;
constexpr int PK_ITERS = 4096;

__global__ void __launch_bounds__(PK_THREADS) pk_ffma(float* out, float s) {
  float a[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) a[j] = s * (threadIdx.x + j);
  const float b = 1.0000001f, c = 1e-7f;
#pragma unroll 1
  for (int i = 0; i < PK_ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 16; ++u)
#pragma unroll
      for (int j = 0; j < 8; ++j) asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(a[j]) : "f"(b), "f"(c));
  }
  float t = 0.f;
#pragma unroll
  for (int j = 0; j < 8; ++j) t += a[j];
  if (t == 1234.5f) out[threadIdx.x] = t;
}

__global__ void __launch_bounds__(PK_THREADS) pk_alu(unsigned* out, unsigned s) {
  unsigned a[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) a[j] = s * (threadIdx.x + j);
  const unsigned y = 0x9E3779B9u, z = 0x7F4A7C15u;
#pragma unroll 1
  for (int i = 0; i < PK_ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 16; ++u)
#pragma unroll
      for (int j = 0; j < 8; ++j) asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(a[j]) : "r"(y), "r"(z));
  }
  unsigned t = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) t ^= a[j];
  if (t == 12345u) out[threadIdx.x] = t;
}

__global__ void __launch_bounds__(PK_THREADS) pk_issue(unsigned* out, unsigned s) {
  float f[4];
  unsigned a[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) { f[j] = 1e-3f * (threadIdx.x + j); a[j] = s * (threadIdx.x + j); }
  const float b = 1.0000001f, c = 1e-7f;
  const unsigned y = 0x9E3779B9u, z = 0x7F4A7C15u;
#pragma unroll 1
  for (int i = 0; i < PK_ITERS; ++i) {
#pragma unroll
    for (int u = 0; u < 16; ++u)
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(f[j]) : "f"(b), "f"(c));
        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(a[j]) : "r"(y), "r"(z));
      }
  }
  unsigned t = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) t ^= a[j] ^ __float_as_uint(f[j]);
  if (t == 12345u) out[threadIdx.x] = t;
}

// best-of-3 seconds of one launch of `k` over grid × PK_THREADS threads
template <class K>
static mdh_status time_best(K k, int grid, void* buf, float* best_ms) {
  cudaEvent_t e0, e1;
  MDH_CUDA(cudaEventCreate(&e0));
  MDH_CUDA(cudaEventCreate(&e1));
  *best_ms = 1e30f;
  for (int r = 0; r < 4; ++r) {       // the first launch warms up (clocks, instruction cache)
    MDH_CUDA(cudaEventRecord(e0));
    k(grid, buf);
    MDH_CUDA(cudaGetLastError());
    MDH_CUDA(cudaEventRecord(e1));
    MDH_CUDA(cudaEventSynchronize(e1));
    float ms = 0.f;
    MDH_CUDA(cudaEventElapsedTime(&ms, e0, e1));
    if (r > 0) *best_ms = std::min(*best_ms, ms);
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return MDH_OK;
}

mdh_status measure_peaks(int device, double* ffma_tflops, double* alu_tops, double* issue_tops) {
  int cur = 0;
  MDH_CUDA(cudaGetDevice(&cur));
  MDH_CUDA(cudaSetDevice(device));
  int sms = 148;
  MDH_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
  const int grid = sms * 4;
  void* buf = nullptr;
  MDH_CUDA(cudaMalloc(&buf, PK_THREADS * sizeof(float)));
  const double threads = (double)grid * PK_THREADS;
  const double per_thread = (double)PK_ITERS * 16 * 8;      // instructions of the timed body
  float ms = 0.f;
  mdh_status s = time_best([](int g, void* b) { pk_ffma<<<g, PK_THREADS>>>((float*)b, 1e-3f); }, grid, buf, &ms);
  if (s == MDH_OK && ffma_tflops) *ffma_tflops = 2.0 * threads * per_thread / (ms * 1e-3) / 1e12;
  if (s == MDH_OK) s = time_best([](int g, void* b) { pk_alu<<<g, PK_THREADS>>>((unsigned*)b, 3u); }, grid, buf, &ms);
  if (s == MDH_OK && alu_tops) *alu_tops = threads * per_thread / (ms * 1e-3) / 1e12;
  if (s == MDH_OK) s = time_best([](int g, void* b) { pk_issue<<<g, PK_THREADS>>>((unsigned*)b, 5u); }, grid, buf, &ms);
  // the issue peak: the best instruction rate any of the kernels sustained (FFMA alone
  // issues one warp-instruction per cycle per SMSP; the FFMA/LOP3 mix does not do better)
  if (s == MDH_OK && issue_tops)
    *issue_tops = std::max(threads * per_thread / (ms * 1e-3) / 1e12, ffma_tflops ? *ffma_tflops / 2.0 : 0.0);
  cudaFree(buf);
  cudaSetDevice(cur);
  return s;
}

}  // namespace mdh
