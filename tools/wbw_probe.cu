// wbw_probe.cu — write-bandwidth probe for the T4 scatter epilogue design (not product code).
// Writes a 20.6 GB fp32 buffer shaped like CCSD(T)'s t3 with different store patterns and
// reports GB/s (CUDA events, best of 5).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o wbw_probe tools/wbw_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int64_t V = 72, O = 24;
constexpr int64_t TOTAL = O * O * O * V * V * V;   // 5 159 780 352 floats

// mode 0: grid-stride, each warp writes 512 contiguous bytes per instruction (float4/lane)
__global__ void seq_v4(float4* p, int64_t n4) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t st = (int64_t)gridDim.x * blockDim.x;
  const float4 v = make_float4(1.f, 2.f, 3.f, 4.f);
  for (; i < n4; i += st) __stcs(p + i, v);
}

// mode 1: "EPI1" pattern — tile = 128 rows (p4 fastest, 72-runs) × 256 cols (p5 stride 72);
// lane = row, one 4-byte store per column: a warp instruction covers 128 contiguous bytes.
// mode 2: "EPI2" pattern — tile = 128 rows (p5, stride 72) × 256 cols (p4 runs of 72);
// thread = row, 8 consecutive columns per 32-byte store: rows 288 B apart per instruction.
// Both map the output as [R][C] blocks with R·C = TOTAL: row-major m-major tiling over
// a virtual (M = 124416, N = 41472) problem where off(m, n) follows t3's layout.
__device__ __forceinline__ int64_t off_epi1(int64_t m, int64_t n) {
  // m = p4 + 72 h1 + 72·24 h2 ; n = p5 + 72 p6 + 72² h3
  const int64_t p4 = m % V, h1 = (m / V) % O, h2 = m / (V * O);
  const int64_t p5 = n % V, p6 = (n / V) % V, h3 = n / (V * V);
  return p4 + V * p5 + V * V * p6 + V * V * V * h1 + V * V * V * O * h2 + V * V * V * O * O * h3;
}
__device__ __forceinline__ int64_t off_epi2(int64_t m, int64_t n) {
  // m = p5 + 72 p6 + 72² h3 ; n = p4 + 72 h1 + 72·24 h2
  return off_epi1(n, m);
}

__global__ void mk_tabs(int64_t* rt, int64_t* ct, int64_t M, int64_t N, int mode) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M + N; i += (int64_t)gridDim.x * blockDim.x) {
    if (i < M) rt[i] = mode == 1 ? off_epi1(i, 0) : off_epi2(i, 0);
    else ct[i - M] = mode == 1 ? off_epi1(0, i - M) : off_epi2(0, i - M);
  }
}

template <int MODE>
__global__ void __launch_bounds__(256, 1) tiles(float* p, int64_t M, int64_t N, const int64_t* rt, const int64_t* ct) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int quad = warp & 3, half = warp >> 2;
  const int64_t tiles_m = M / 128, tiles_n = N / 256, T = tiles_m * tiles_n;
  const int64_t t0 = (int64_t)blockIdx.x * T / gridDim.x, t1 = (int64_t)(blockIdx.x + 1) * T / gridDim.x;
  for (int64_t t = t0; t < t1; ++t) {
    const int64_t nb = t / tiles_m, mb = t % tiles_m;
    const int64_t m = mb * 128 + quad * 32 + lane;
    const int64_t ro = __ldg(rt + m);
    for (int c = 0; c < 4; ++c) {
      const int64_t n0 = nb * 256 + half * 128 + c * 32;
      if (MODE == 1) {
#pragma unroll 8
        for (int j = 0; j < 32; ++j) __stcs(p + ro + __ldg(ct + n0 + j), (float)j);
      } else {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          float* q = p + ro + __ldg(ct + n0 + 8 * j);
          asm volatile("st.global.cs.v8.f32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1};" ::"l"(q), "f"(1.f) : "memory");
        }
      }
    }
  }
}

// mode 3: smem-staged TMA bulk stores: each CTA owns contiguous 36 KB chunks (one 72-run
// block of 128 rows), fills smem with st.shared, then one thread issues cp.async.bulk
__global__ void __launch_bounds__(256, 1) bulk(float* p, int64_t nchunks, int chunk_floats) {
  extern __shared__ __align__(128) float sm[];
  const int64_t c0 = (int64_t)blockIdx.x * nchunks / gridDim.x, c1 = (int64_t)(blockIdx.x + 1) * nchunks / gridDim.x;
  int buf = 0;
  for (int64_t c = c0; c < c1; ++c, buf ^= 1) {
    float* s = sm + buf * chunk_floats;
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
    __syncthreads();
    for (int i = threadIdx.x; i < chunk_floats; i += blockDim.x) s[i] = (float)i;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (threadIdx.x == 0) {
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(p + c * chunk_floats),
                   "r"((uint32_t)__cvta_generic_to_shared(s)), "r"(chunk_floats * 4)
                   : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
  }
  if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// mode 4: per-warp staging like the T4 EPI 3 epilogue: each warp fills a 32×72-float piece
// (9 KB) with st.shared and issues its own cp.async.bulk; NB buffers per warp
template <int NB>
__global__ void __launch_bounds__(256, 1) bulk_warp(float* p, int64_t npieces, int piece_floats) {
  extern __shared__ __align__(128) float sm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t gw = (int64_t)blockIdx.x * 8 + warp, nw = (int64_t)gridDim.x * 8;
  const int64_t c0 = gw * npieces / nw, c1 = (gw + 1) * npieces / nw;
  float* mine = sm + (size_t)warp * NB * piece_floats;
  int b = 0;
  for (int64_t c = c0; c < c1; ++c) {
    float* s = mine + b * piece_floats;
    if (lane == 0) {
      if (NB == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      else asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
    }
    __syncwarp();
    for (int i = lane * 4; i < piece_floats; i += 128)
      *reinterpret_cast<float4*>(s + i) = make_float4(1.f, 2.f, 3.f, (float)i);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
    if (lane == 0) {
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(p + c * piece_floats),
                   "r"((uint32_t)__cvta_generic_to_shared(s)), "r"(piece_floats * 4)
                   : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
    if (NB == 2) b ^= 1;
  }
  if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main() {
  float* p;
  if (cudaMalloc(&p, TOTAL * 4) != cudaSuccess) { printf("alloc failed\n"); return 1; }
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto run = [&](const char* name, auto launch) {
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
      cudaEventRecord(a);
      launch();
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (r > 0 && ms < best) best = ms;
    }
    cudaError_t e = cudaGetLastError();
    printf("%-40s %8.3f ms  %7.1f GB/s  %s\n", name, best, TOTAL * 4.0 / (best * 1e-3) / 1e9, cudaGetErrorString(e));
  };
  const int64_t M = V * O * O * 3 / 3, N = O * V * V;   // M = 41472 (epi1 rows), N = 124416
  run("seq float4, 148x256 (8 warps/SM)", [&] { seq_v4<<<sms, 256>>>((float4*)p, TOTAL / 4); });
  run("seq float4, 148x512 (16 warps/SM)", [&] { seq_v4<<<sms, 512>>>((float4*)p, TOTAL / 4); });
  run("seq float4, 148x1024 (32 warps/SM)", [&] { seq_v4<<<sms, 1024>>>((float4*)p, TOTAL / 4); });
  run("seq float4, 4x148x1024", [&] { seq_v4<<<4 * sms, 1024>>>((float4*)p, TOTAL / 4); });
  int64_t *rt, *ct;
  cudaMalloc(&rt, (M + N) * 8);
  cudaMalloc(&ct, (M + N) * 8);
  mk_tabs<<<1024, 256>>>(rt, ct, M, N, 1);
  run("EPI1 pattern (lane=row, 4 B)", [&] { tiles<1><<<sms, 256>>>(p, M, N, rt, ct); });
  mk_tabs<<<1024, 256>>>(rt, ct, N, M, 2);
  run("EPI2 pattern (thread=row, 32 B)", [&] { tiles<2><<<sms, 256>>>(p, N, M, rt, ct); });
  run("EPI2 pattern, 2 CTAs/SM", [&] { tiles<2><<<2 * sms, 256>>>(p, N, M, rt, ct); });
  const int chunk = 128 * 72;   // 36 KB
  cudaFuncSetAttribute(bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * chunk * 4);
  run("bulk 36KB chunks, smem staged", [&] { bulk<<<sms, 256, 2 * chunk * 4>>>(p, TOTAL / chunk, chunk); });
  cudaFuncSetAttribute(bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * 2 * chunk * 4);
  run("bulk 72KB chunks, smem staged", [&] { bulk<<<sms, 256, 2 * 2 * chunk * 4>>>(p, TOTAL / (2 * chunk), 2 * chunk); });
  const int piece = 32 * 72;
  cudaFuncSetAttribute(bulk_warp<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16 * piece * 4);
  cudaFuncSetAttribute(bulk_warp<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * piece * 4);
  run("per-warp 9KB pieces, 2 buffers", [&] { bulk_warp<2><<<sms, 256, 16 * piece * 4>>>(p, TOTAL / piece, piece); });
  run("per-warp 9KB pieces, 1 buffer", [&] { bulk_warp<1><<<sms, 256, 8 * piece * 4>>>(p, TOTAL / piece, piece); });
  return 0;
}
