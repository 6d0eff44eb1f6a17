// t1_stencil.cu — T1: all-cc md_hom (no pw dims): maps and stencils (Jacobi1D/3D,
// Gaussian; Fig 3, Listing 10 caption P:308, 3-access example P:251).
//
// Every cc dim maps to the grid (A1): the innermost iteration dim to threadIdx.x (the
// contiguous dim of the buffers: 128-byte coalesced warp accesses), the next one to
// threadIdx.y, and the outermost is marched by each thread over a z-chunk so that the
// planes a stencil re-reads (z±1, y±1, x±1) are served from L1/L2 and every input
// element comes from HBM about once (A2); f = Σ_a w_a·x_a (reading C-16) in fp32
// with FMA (reading C-13).  HBM-bound: ≈8.05 B per output point for Jacobi3D.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <mutex>
#include <type_traits>
#include <vector>

#include "kcommon.cuh"

namespace mdh {

constexpr int T1_MAX_ACC = 32;

struct T1Params {
  const void* ptr[T1_MAX_ACC];
  int64_t base[T1_MAX_ACC];
  float w[T1_MAX_ACC];
  int nacc, f, dt, odt;
  int64_t Lz[T1_MAX_ACC], Ly[T1_MAX_ACC], Lx[T1_MAX_ACC];   // per access
  int64_t oLz, oLy, oLx, obase;
  int64_t Z, Y, X;
  int zchunk;
  void* out;
};

template <int NACC, int F, bool SAME_L>
__global__ void __launch_bounds__(256) t1_kernel(const __grid_constant__ T1Params P) {
  const int nacc = NACC > 0 ? NACC : P.nacc;
  const int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t y = (int64_t)blockIdx.y * blockDim.y + threadIdx.y;
  if (x >= P.X || y >= P.Y) return;
  const int64_t z0 = (int64_t)blockIdx.z * P.zchunk;
  const int64_t z1 = min(P.Z, z0 + P.zchunk);
  const float* in0 = (const float*)P.ptr[0];
  float w[NACC > 0 ? NACC : T1_MAX_ACC];
  int64_t off[NACC > 0 ? NACC : T1_MAX_ACC];
#pragma unroll
  for (int a = 0; a < (NACC > 0 ? NACC : T1_MAX_ACC); ++a) {
    if (a < nacc) {
      w[a] = P.w[a];
      off[a] = P.base[a] + y * P.Ly[a] + x * P.Lx[a] + z0 * P.Lz[a];
    }
  }
  int64_t oo = P.obase + y * P.oLy + x * P.oLx + z0 * P.oLz;
  for (int64_t z = z0; z < z1; ++z) {
    float acc;
    if (F == MDH_F_STENCIL) {
      acc = w[0] * __ldg(in0 + off[0]);
#pragma unroll
      for (int a = 1; a < (NACC > 0 ? NACC : T1_MAX_ACC); ++a)
        if (a < nacc) acc = fmaf(w[a], __ldg((SAME_L ? in0 : (const float*)P.ptr[a]) + off[a]), acc);
    } else if (F == MDH_F_MUL) {
      acc = __ldg(in0 + off[0]) * __ldg((const float*)P.ptr[1] + off[1]);
    } else {
      acc = __ldg(in0 + off[0]);
    }
    store_as<float>(P.out, P.odt, oo, acc);
#pragma unroll
    for (int a = 0; a < (NACC > 0 ? NACC : T1_MAX_ACC); ++a)
      if (a < nacc) off[a] += P.Lz[a];
    oo += P.oLz;
  }
}

// ---- specialised 7-point cross (radius 1, "j3d7pt", reading C-16) ----------------------
// Each thread owns 4 consecutive x outputs of one y row and marches z.  The centre row
// segment (x0-1 … x0+4) of planes z-1, z, z+1 lives in a register queue, so a z step
// loads only the new centre row of plane z+1 plus the y-1 / y+1 rows of plane z — six
// 128/64-bit loads per 4 outputs (instead of 28 scalar loads); x±1 come from the centre
// row registers.  Every input element is read from HBM once (the y±1 re-reads of
// neighbouring threads hit L1/L2).
struct J7Params {
  const float* u;
  float* v;
  int64_t bc;              // element offset of the centre access at the origin
  int64_t Ly, Lz;          // input strides of y and z (x stride 1)
  int64_t ob, oLy, oLz;    // output (x stride 1)
  int X, Y, Z, zchunk;
  float wc, wxm, wxp, wym, wyp, wzm, wzp;
  // fused halo exchange (stencil time-stepping, reading C-34): the outputs of the first /
  // last iteration plane are also stored into the lower / upper neighbour's halo plane
  // (peer device memory: same GPU, NVLink P2P or CUDA-IPC mapped) at in-plane offset
  // hbase + x + y·oLy; NULL = no neighbour
  float* hlo;
  float* hhi;
  int64_t hbase;
};

// 16- / 8-byte read-only loads with an optional L2 prefetch-size hint (PF 1: 128 B, 2: 256 B
// — the L2 fetches the whole aligned sector group from HBM on a miss)
template <int PF>
__device__ __forceinline__ float4 ldv4(const float* p) {
  float4 a;
  if (PF == 2)
    asm volatile("ld.global.nc.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w) : "l"(p));
  else if (PF == 1)
    asm volatile("ld.global.nc.L2::128B.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w) : "l"(p));
  else
    a = __ldg(reinterpret_cast<const float4*>(p));
  return a;
}
template <int PF>
__device__ __forceinline__ float2 ldv2(const float* p) {
  float2 a;
  if (PF == 2)
    asm volatile("ld.global.nc.L2::256B.v2.f32 {%0,%1}, [%2];" : "=f"(a.x), "=f"(a.y) : "l"(p));
  else if (PF == 1)
    asm volatile("ld.global.nc.L2::128B.v2.f32 {%0,%1}, [%2];" : "=f"(a.x), "=f"(a.y) : "l"(p));
  else
    a = __ldg(reinterpret_cast<const float2*>(p));
  return a;
}

// r[k] = p[k], k = 0..NX+1 (p = the x0-1 position, 16-byte aligned when VEC); rem = the
// number of valid positions
template <bool VEC, int NX, int PF = 0>
__device__ __forceinline__ void rowq(const float* p, bool full, int64_t rem, float* r) {
  if (VEC && full) {
#pragma unroll
    for (int q = 0; q < NX / 4; ++q) {
      const float4 a = ldv4<PF>(p + 4 * q);
      r[4 * q] = a.x; r[4 * q + 1] = a.y; r[4 * q + 2] = a.z; r[4 * q + 3] = a.w;
    }
    const float2 b = ldv2<PF>(p + NX);
    r[NX] = b.x; r[NX + 1] = b.y;
  } else {
#pragma unroll
    for (int k = 0; k < NX + 2; ++k) r[k] = k < rem ? __ldg(p + k) : 0.f;
  }
}
// VEC_OUT: 0 scalar stores; 1 8-byte stores (even output base); 2 odd output base
// (e.g. the same-shape sweep of reading C-34, v[z+1,y+1,x+1]): scalar, 8-byte…, scalar.
// NX: x outputs per thread (4, or 8 with tile knob vec=8)
template <bool VEC_IN, int VEC_OUT, int NX, int PF = 0>
__global__ void __launch_bounds__(128) t1_j3d7_kernel(const __grid_constant__ J7Params P) {
  // stencil time-stepping launches sweep t+1 as a programmatic dependent of sweep t: wait
  // for the previous sweep's writes (a no-op for a plain launch), then let the next sweep's
  // blocks be scheduled as this grid's SM slots free up
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int x0 = (blockIdx.x * blockDim.x + threadIdx.x) * NX;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  if (x0 >= P.X || y >= P.Y) return;
  const int z0 = blockIdx.z * P.zchunk;
  const int z1 = min(P.Z, z0 + P.zchunk);
  const bool full = x0 + NX <= P.X;
  const int64_t rem = (int64_t)P.X + 1 - x0 + 1;     // valid positions x0-1 … X (centre-relative)
  const float* pc = P.u + P.bc - 1 + x0 + (int64_t)y * P.Ly + (int64_t)z0 * P.Lz;
  float* po = P.v + P.ob + x0 + (int64_t)y * P.oLy + (int64_t)z0 * P.oLz;
  float rm[NX + 2], r0[NX + 2], rp[NX + 2], ym[NX + 2], yp[NX + 2];
  rowq<VEC_IN, NX, PF>(pc - P.Lz, full, rem, rm);
  rowq<VEC_IN, NX, PF>(pc, full, rem, r0);
  for (int z = z0; z < z1; ++z) {
    rowq<VEC_IN, NX, PF>(pc + P.Lz, full, rem, rp);
    rowq<VEC_IN, NX, PF>(pc - P.Ly, full, rem, ym);
    rowq<VEC_IN, NX, PF>(pc + P.Ly, full, rem, yp);
    float o[NX];
#pragma unroll
    for (int j = 0; j < NX; ++j) {
      float acc = P.wc * r0[j + 1];
      acc = fmaf(P.wxm, r0[j], acc);
      acc = fmaf(P.wxp, r0[j + 2], acc);
      acc = fmaf(P.wym, ym[j + 1], acc);
      acc = fmaf(P.wyp, yp[j + 1], acc);
      acc = fmaf(P.wzm, rm[j + 1], acc);
      acc = fmaf(P.wzp, rp[j + 1], acc);
      o[j] = acc;
    }
    // streaming (evict-first) stores: the output is never re-read, so it should not push
    // the input rows that neighbouring CTAs still read (their y±1 rows) out of L2
    if (VEC_OUT == 1 && full) {
#pragma unroll
      for (int j = 0; j < NX; j += 2) __stcs(reinterpret_cast<float2*>(po + j), make_float2(o[j], o[j + 1]));
    } else if (VEC_OUT == 2 && full) {
      __stcs(po, o[0]);
#pragma unroll
      for (int j = 1; j + 1 < NX; j += 2) __stcs(reinterpret_cast<float2*>(po + j), make_float2(o[j], o[j + 1]));
      __stcs(po + NX - 1, o[NX - 1]);
    } else {
#pragma unroll
      for (int j = 0; j < NX; ++j)
        if (x0 + j < P.X) po[j] = o[j];
    }
    // this plane may also be a neighbour's halo plane: the first owned plane goes to the
    // lower neighbour, the last to the upper one (a one-plane slab feeds both); the two
    // stores are independent, so a rank with only one neighbour still writes its halo
    if (z == 0 && P.hlo) {
      float* q = P.hlo + P.hbase + x0 + (int64_t)y * P.oLy;
#pragma unroll
      for (int j = 0; j < NX; ++j)
        if (x0 + j < P.X) q[j] = o[j];
    }
    if (z == P.Z - 1 && P.hhi) {
      float* q = P.hhi + P.hbase + x0 + (int64_t)y * P.oLy;
#pragma unroll
      for (int j = 0; j < NX; ++j)
        if (x0 + j < P.X) q[j] = o[j];
    }
#pragma unroll
    for (int k = 0; k < NX + 2; ++k) { rm[k] = r0[k]; r0[k] = rp[k]; }
    pc += P.Lz;
    po += P.oLz;
  }
}

// ---- TMA-staged 7-point cross (tile knob stages = ring depth ≥ 3) --------------------
// A CTA owns a 128 × 32 (x × y) output tile and marches z over a z-chunk.  A producer warp
// streams the input planes the chunk needs — a 132 × 34 box per plane, one
// cp.async.bulk.tensor.3d each — into a ring of `stages` shared-memory planes (mbarrier
// complete_tx), so several planes per CTA are in flight without holding registers; eight
// compute warps read each output plane's 7 taps from the three resident input planes and
// free the oldest plane as they finish.  The box starts one column left of the tile's first
// centre (TMA box coordinates must be non-negative on this part: a negative start faults),
// so a lane's row segment (left, 4 centres, right) is one aligned LDS.128 + LDS.64 and the
// other taps an LDS.128 + LDS.32 each.  Box elements past the tensor end are zero-filled by
// the TMA unit and never stored.
constexpr int J7T_TX = 128, J7T_TY = 32, J7T_BX = 132, J7T_BY = J7T_TY + 2;
constexpr int J7T_PLANE = J7T_BX * J7T_BY * 4;       // 9792 bytes loaded per plane
constexpr int J7T_SLOT = (J7T_PLANE + 127) / 128 * 128;   // ring slot (TMA destinations 128-byte aligned)
constexpr int J7T_THREADS = 288;                     // 8 compute warps + 1 producer warp
constexpr int J7T_MAXS = 8;

__device__ __forceinline__ void j7t_mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(bar),
      "r"(parity)
      : "memory");
}

template <int VEC_OUT>
__global__ void __launch_bounds__(J7T_THREADS) t1_j3d7_tma_kernel(const __grid_constant__ CUtensorMap map,
                                                                  const __grid_constant__ J7Params P,
                                                                  int stages, int cx, int cy, int cz, int ny) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  extern __shared__ __align__(1024) uint8_t j7t_raw[];
  float* sm = (float*)(j7t_raw + ((1024u - ((uint32_t)__cvta_generic_to_shared(j7t_raw) & 1023u)) & 1023u));
  __shared__ __align__(8) uint64_t bar_full[J7T_MAXS], bar_empty[J7T_MAXS];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int xb = blockIdx.x * J7T_TX, yb = blockIdx.y * J7T_TY;
  const int z0 = blockIdx.z * P.zchunk, z1 = min(P.Z, z0 + P.zchunk);
  const int nplanes = z1 - z0 + 2;                   // input planes z0 .. z1+1
  const uint32_t sfull = (uint32_t)__cvta_generic_to_shared(bar_full);
  const uint32_t sempty = (uint32_t)__cvta_generic_to_shared(bar_empty);
  if (tid == 0) {
    for (int s = 0; s < stages; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sfull + 8 * s));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 256;" ::"r"(sempty + 8 * s));
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == 8) {
    // ---- producer: plane j into slot j % stages (waits for the consumers to free it)
    if (lane == 0) {
      const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
      for (int j = 0; j < nplanes; ++j) {
        const int s = j % stages;
        if (j >= stages) j7t_mbar_wait(sempty + 8 * s, ((j / stages) - 1) & 1);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sfull + 8 * s), "r"(J7T_PLANE)
                     : "memory");
        // the input viewed as 2-D rows [nz·ny][nx]: the box's 18 rows are rows yb+cy-1 … of
        // plane z (rows past the plane end belong to the next plane — never stored)
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
            ::"r"(base + s * J7T_SLOT), "l"((uint64_t)&map), "r"(sfull + 8 * s), "r"(xb + cx - 1),
            "r"((z0 + j + cz - 1) * ny + yb + cy - 1)
            : "memory");
      }
    }
  } else {
  // ---- compute: warp w owns tile rows w, w + 8, …, lane l the outputs x = xb + 4l … +3
  const int x = xb + 4 * lane;
  const int nx = min(4, P.X - x);                    // valid outputs of this lane (≤ 0: none)
  j7t_mbar_wait(sfull, 0);
  j7t_mbar_wait(sfull + 8 * (1 % stages), (1 / stages) & 1);
  for (int z = z0; z < z1; ++z) {
    const int j = z - z0;
    j7t_mbar_wait(sfull + 8 * ((j + 2) % stages), ((j + 2) / stages) & 1);
    const float* pm = sm + (size_t)(j % stages) * (J7T_SLOT / 4);
    const float* p0 = sm + (size_t)((j + 1) % stages) * (J7T_SLOT / 4);
    const float* pp = sm + (size_t)((j + 2) % stages) * (J7T_SLOT / 4);
#pragma unroll
    for (int h = 0; h < J7T_TY / 8; ++h) {
      const int ty = warp + 8 * h, y = yb + ty;
      const int c = (ty + 1) * J7T_BX + 4 * lane;        // the left neighbour of output x in the box
      const float4 ra = *reinterpret_cast<const float4*>(p0 + c);
      const float2 rb = *reinterpret_cast<const float2*>(p0 + c + 4);
      const float4 yma = *reinterpret_cast<const float4*>(p0 + c - J7T_BX);
      const float4 ypa = *reinterpret_cast<const float4*>(p0 + c + J7T_BX);
      const float4 zma = *reinterpret_cast<const float4*>(pm + c);
      const float4 zpa = *reinterpret_cast<const float4*>(pp + c);
      const float rr[6] = {ra.x, ra.y, ra.z, ra.w, rb.x, rb.y};
      const float ymv[4] = {yma.y, yma.z, yma.w, p0[c - J7T_BX + 4]}, ypv[4] = {ypa.y, ypa.z, ypa.w, p0[c + J7T_BX + 4]};
      const float zmv[4] = {zma.y, zma.z, zma.w, pm[c + 4]}, zpv[4] = {zpa.y, zpa.z, zpa.w, pp[c + 4]};
      float o[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        float acc = P.wc * rr[k + 1];
        acc = fmaf(P.wxm, rr[k], acc);
        acc = fmaf(P.wxp, rr[k + 2], acc);
        acc = fmaf(P.wym, ymv[k], acc);
        acc = fmaf(P.wyp, ypv[k], acc);
        acc = fmaf(P.wzm, zmv[k], acc);
        acc = fmaf(P.wzp, zpv[k], acc);
        o[k] = acc;
      }
      if (y < P.Y && nx > 0) {
        float* po = P.v + P.ob + x + (int64_t)y * P.oLy + (int64_t)z * P.oLz;
        if (VEC_OUT == 1 && nx == 4) {
          __stcs(reinterpret_cast<float2*>(po), make_float2(o[0], o[1]));
          __stcs(reinterpret_cast<float2*>(po + 2), make_float2(o[2], o[3]));
        } else if (VEC_OUT == 2 && nx == 4) {
          __stcs(po, o[0]);
          __stcs(reinterpret_cast<float2*>(po + 1), make_float2(o[1], o[2]));
          __stcs(po + 3, o[3]);
        } else {
#pragma unroll
          for (int k = 0; k < 4; ++k)
            if (k < nx) po[k] = o[k];
        }
        if (z == 0 && P.hlo) {
          float* q = P.hlo + P.hbase + x + (int64_t)y * P.oLy;
#pragma unroll
          for (int k = 0; k < 4; ++k)
            if (k < nx) q[k] = o[k];
        }
        if (z == P.Z - 1 && P.hhi) {
          float* q = P.hhi + P.hbase + x + (int64_t)y * P.oLy;
#pragma unroll
          for (int k = 0; k < 4; ++k)
            if (k < nx) q[k] = o[k];
        }
      }
    }
    // input plane j is not needed by later output planes: free its slot
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sempty + 8 * (j % stages)) : "memory");
  }
  }
  __syncthreads();
}

// ---- dense 2-D box stencil (H×W window, e.g. Gaussian_2D 5×5, Fig 3) -------
// Each thread owns 4 consecutive x outputs and marches y over a y-chunk with a register
// window of the last H input rows (4+W-1 values each): a y step loads ONE new row segment
// (two 16-byte loads for W = 5) and does 4·|accesses| FMAs; rows are re-read only across
// chunk boundaries (H-1 halo rows per chunk, L2 hits).  Absent window taps (a sparse
// stencil inside its bounding box) are skipped through the mask, so the arithmetic is
// exactly Σ_a w_a·x_a over the spec's accesses (reading C-16/C-31), fp32 FMA.
struct Box2Params {
  const float* u;
  float* v;
  int64_t b0;              // element offset of window tap (0,0) at the origin
  int64_t Ly;              // input row stride (x stride 1)
  int64_t ob, oLy;         // output (x stride 1)
  int X, Y, ychunk;
  uint64_t mask;           // bit r*W+s: tap (r,s) present
  float w[49];             // w[r*W+s]
};

// MINB = 8 CTAs of 128 threads per SM: the compiler fits the 5×5 window ring in 64 registers
// without spilling (78 unconstrained → 6 CTAs/SM); Gaussian_2D 4096² 0.0348 → 0.0327 ms on
// one box (the kernel is memory-latency bound: more resident rows in flight)
template <int H, int W, bool DENSE, int MINB = 8>
__global__ void __launch_bounds__(128, MINB) t1_box2d_kernel(const __grid_constant__ Box2Params P) {
  constexpr int NW = 4 + W - 1;
  const int x0 = (blockIdx.x * blockDim.x + threadIdx.x) * 4;
  if (x0 >= P.X) return;
  const int y0 = blockIdx.y * P.ychunk;
  const int y1 = min(P.Y, y0 + P.ychunk);
  const int nv = min(4, P.X - x0);                       // valid outputs of this thread
  const bool vec = nv == 4 && ((P.b0 + x0) & 3) == 0 && (P.Ly & 3) == 0;
  const bool ovec = nv == 4 && ((P.ob + x0) & 3) == 0 && (P.oLy & 3) == 0;
  const float* pin = P.u + P.b0 + x0 + (int64_t)y0 * P.Ly;
  float* po = P.v + P.ob + x0 + (int64_t)y0 * P.oLy;
  float w[H * W];
#pragma unroll
  for (int k = 0; k < H * W; ++k) w[k] = P.w[k];
  // window ring: slot (ph + r) % H holds window row r at phase ph; unrolling the y loop by H
  // makes every slot index a compile-time constant (no register moves)
  float win[H][NW];
  auto load_row = [&](const float* p, float* r) {
    if (vec) {
#pragma unroll
      for (int k = 0; k + 4 <= NW; k += 4) {
        const float4 a = __ldg(reinterpret_cast<const float4*>(p + k));
        r[k] = a.x; r[k + 1] = a.y; r[k + 2] = a.z; r[k + 3] = a.w;
      }
      if (NW % 4 >= 2) {
        const float2 a = __ldg(reinterpret_cast<const float2*>(p + (NW & ~3)));
        r[NW & ~3] = a.x; r[(NW & ~3) + 1] = a.y;
      }
      if (NW % 2) r[NW - 1] = __ldg(p + NW - 1);
    } else {
#pragma unroll
      for (int k = 0; k < NW; ++k) r[k] = k < nv + W - 1 ? __ldg(p + k) : 0.f;
    }
  };
  // step at phase PH: load window row H-1 into slot (PH + H - 1) % H, compute, store
  auto step = [&](auto ph) {
    constexpr int PH = decltype(ph)::value;
    load_row(pin + (int64_t)(H - 1) * P.Ly, win[(PH + H - 1) % H]);
    float o[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int r = 0; r < H; ++r)
#pragma unroll
      for (int s = 0; s < W; ++s)
        if (DENSE || ((P.mask >> (r * W + s)) & 1))
#pragma unroll
          for (int j = 0; j < 4; ++j) o[j] = fmaf(w[r * W + s], win[(PH + r) % H][j + s], o[j]);
    if (ovec) {
      *reinterpret_cast<float4*>(po) = make_float4(o[0], o[1], o[2], o[3]);
    } else {
#pragma unroll
      for (int j = 0; j < 4; ++j)
        if (j < nv) po[j] = o[j];
    }
    pin += P.Ly;
    po += P.oLy;
  };
#pragma unroll
  for (int r = 0; r < H - 1; ++r) load_row(pin + (int64_t)r * P.Ly, win[r]);
  int y = y0;
  for (; y + H <= y1; y += H) {
    step(std::integral_constant<int, 0>{});
    step(std::integral_constant<int, 1>{});
    step(std::integral_constant<int, 2>{});
    if constexpr (H > 3) {
      step(std::integral_constant<int, 3>{});
      step(std::integral_constant<int, 4>{});
    }
  }
  // tail (< H rows): phases 0, 1, … continue the ring from phase 0
  if (y < y1) step(std::integral_constant<int, 0>{});
  if (y + 1 < y1) step(std::integral_constant<int, 1>{});
  if constexpr (H > 3) {
    if (y + 2 < y1) step(std::integral_constant<int, 2>{});
    if (y + 3 < y1) step(std::integral_constant<int, 3>{});
  }
}

// Recognise a dense 2-D window: one fp32 input buffer, ≤ 49 accesses sharing the linear
// part with x stride 1, taps inside an H×W box, H = W ∈ {3, 5}; exactly two non-degenerate
// dims (y, x).  auxi = {-2, dy, dx, H, W, b0, tap index per access ...}.
static bool detect_box2d(Plan* p) {
  if (p->n_in != 1 || p->f != MDH_F_STENCIL || p->in[0].dtype != MDH_F32 || p->out[0].dtype != MDH_F32) return false;
  int dims[2], nd = 0;
  for (int d = 0; d < p->D; ++d)
    if (p->size[d] > 1) { if (nd == 2) return false; dims[nd++] = d; }
  if (nd != 2) return false;
  const int dy = dims[0], dx = dims[1];
  const Buf& B = p->in[0];
  for (int a = 1; a < B.nacc; ++a)
    for (int d = 0; d < p->D; ++d)
      if (B.acc[a].L[d] != B.acc[0].L[d]) return false;
  const int64_t Ly = B.acc[0].L[dy];
  if (B.acc[0].L[dx] != 1 || Ly < 8 || p->out[0].acc[0].L[dx] != 1) return false;
  // decompose each tap offset relative to the smallest base into (r, s), 0 <= s < Ly/2
  int64_t bmin = INT64_MAX;
  for (int a = 0; a < B.nacc; ++a) bmin = std::min(bmin, B.acc[a].base);
  int rmin = 1 << 30, rmax = -1, smin = 1 << 30, smax = -(1 << 30);
  std::vector<std::pair<int64_t, int64_t>> rs;
  for (int a = 0; a < B.nacc; ++a) {
    const int64_t d = B.acc[a].base - bmin;
    int64_t r = (d + Ly / 2) / Ly, s = d - r * Ly;
    rs.push_back({r, s});
    rmin = std::min<int>(rmin, (int)r); rmax = std::max<int>(rmax, (int)r);
    smin = std::min<int>(smin, (int)s); smax = std::max<int>(smax, (int)s);
  }
  const int H = rmax - rmin + 1, W = smax - smin + 1;
  if (!((H == 3 && W == 3) || (H == 5 && W == 5)) || B.nacc < 4) return false;
  std::vector<int> seen(H * W, 0);
  p->auxi = {-2, dy, dx, H, W, bmin + rmin * Ly + smin};
  for (auto& t : rs) {
    const int k = (int)(t.first - rmin) * W + (int)(t.second - smin);
    if (seen[k]++) return false;              // duplicate tap: keep the literal generic path
    p->auxi.push_back(k);
  }
  return true;
}

static mdh_status launch_box2d(const Plan& p, const void* const* in, void* const* out, cudaStream_t st) {
  Box2Params P;
  memset(&P, 0, sizeof(P));
  const int dy = (int)p.auxi[1], dx = (int)p.auxi[2], H = (int)p.auxi[3], W = (int)p.auxi[4];
  const Buf& B = p.in[0];
  const Access& O = p.out[0].acc[0];
  P.u = (const float*)in[0];
  P.v = (float*)out[0];
  P.b0 = p.auxi[5];
  P.Ly = B.acc[0].L[dy];
  P.ob = O.base;
  P.oLy = O.L[dy];
  P.X = (int)p.size[dx];
  P.Y = (int)p.size[dy];
  for (int a = 0; a < B.nacc; ++a) {
    const int k = (int)p.auxi[6 + a];
    P.mask |= 1ull << k;
    P.w[k] = (float)p.fparams[a];
  }
  // y-chunk: forced tile knob zchunk, else 16 rows (measured 30.8 µs at 4096², 32: 31.7, 64: 47) (the table's T1 entries are Jacobi's z-chunks)
  int yc = p.tiles.source.find("forced") != std::string::npos && p.tiles.zchunk > 0 ? p.tiles.zchunk : 16;
  if (yc > P.Y) yc = P.Y;
  P.ychunk = yc;
  const int tx = 64;
  dim3 grid((unsigned)((P.X + 4 * tx - 1) / (4 * tx)), (unsigned)((P.Y + yc - 1) / yc));
  const bool dense = P.mask == (H * W == 64 ? ~0ull : (1ull << (H * W)) - 1);
  if (H == 5 && dense && p.tiles.mode == 1) t1_box2d_kernel<5, 5, true, 1><<<grid, tx, 0, st>>>(P);   // unconstrained
  else if (H == 5 && dense) t1_box2d_kernel<5, 5, true><<<grid, tx, 0, st>>>(P);
  else if (H == 5) t1_box2d_kernel<5, 5, false><<<grid, tx, 0, st>>>(P);
  else if (dense) t1_box2d_kernel<3, 3, true><<<grid, tx, 0, st>>>(P);
  else t1_box2d_kernel<3, 3, false><<<grid, tx, 0, st>>>(P);
  (void)W;
  return post_launch("t1_box2d_kernel");
}

// Recognise the 7-point cross: one fp32 input buffer, 7 accesses sharing the linear part
// (x stride 1), shifts = centre ± one unit in exactly one of x, y, z.  Stores in auxi:
// [dz_dim, dy_dim, dx_dim, centre access, index of access for xm,xp,ym,yp,zm,zp].
static bool detect_j3d7(Plan* p) {
  if (p->n_in != 1 || p->in[0].nacc != 7 || p->in[0].dtype != MDH_F32 || p->f != MDH_F_STENCIL) return false;
  if (p->out[0].dtype != MDH_F32) return false;
  int dims[3], nd = 0;
  for (int d = 0; d < p->D; ++d)
    if (p->size[d] > 1) { if (nd == 3) return false; dims[nd++] = d; }
  if (nd != 3) return false;
  const int dz = dims[0], dy = dims[1], dx = dims[2];
  const Buf& B = p->in[0];
  for (int a = 1; a < 7; ++a)
    for (int d = 0; d < p->D; ++d)
      if (B.acc[a].L[d] != B.acc[0].L[d]) return false;
  const int64_t Lx = B.acc[0].L[dx], Ly = B.acc[0].L[dy], Lz = B.acc[0].L[dz];
  if (Lx != 1 || Ly < 4 || Lz < 3 * Ly) return false;
  const Access& O = p->out[0].acc[0];
  if (O.L[dx] != 1) return false;
  for (int c = 0; c < 7; ++c) {
    int idx[6] = {-1, -1, -1, -1, -1, -1};
    bool ok = true;
    for (int a = 0; a < 7 && ok; ++a) {
      if (a == c) continue;
      int64_t s = B.acc[a].base - B.acc[c].base;
      int k = s == -1 ? 0 : s == 1 ? 1 : s == -Ly ? 2 : s == Ly ? 3 : s == -Lz ? 4 : s == Lz ? 5 : -1;
      if (k < 0 || idx[k] >= 0) ok = false; else idx[k] = a;
    }
    if (!ok) continue;
    p->auxi = {dz, dy, dx, c, idx[0], idx[1], idx[2], idx[3], idx[4], idx[5]};
    return true;
  }
  return false;
}

mdh_status prepare_t1(Plan* p) {
  p->auxi.clear();
  if (detect_j3d7(p)) {
    p->ws_kernel = 0;
    p->t4_variant = 0;
    const Buf& B = p->in[0];
    const int64_t Ly = B.acc[p->auxi[3]].L[p->auxi[1]], Lz = B.acc[p->auxi[3]].L[p->auxi[0]];
    const bool tma = p->tiles.stages >= 3 && B.rank == 3 && B.shape[2] == Ly && B.shape[1] * B.shape[2] == Lz &&
                     Ly % 4 == 0 && Lz % 4 == 0;
    p->why += tma ? " [7-point cross, tma-staged plane ring]" : " [7-point cross register-queue kernel]";
    return MDH_OK;
  }
  if (detect_box2d(p)) {
    p->ws_kernel = 0;
    p->why += " [2-D box-window register kernel]";
    return MDH_OK;
  }
  // fast path: fp32 inputs, <= 3 non-degenerate dims, <= 32 accesses; else generic
  bool ok = p->compute == MDH_F32 && p->n_in_acc <= T1_MAX_ACC && p->n_out == 1 && p->out[0].nacc == 1;
  for (int b = 0; b < p->n_in; ++b) ok &= p->in[b].dtype == MDH_F32;
  int nd = 0;
  for (int d = 0; d < p->D; ++d) nd += p->size[d] > 1;
  ok &= nd <= 3;
  if (!ok) {
    p->tmpl = T0_GENERIC;
    p->why = "all-cc map outside the T1 fast path: generic template";
    return prepare_t0(p);
  }
  p->ws_kernel = 0;
  return MDH_OK;
}

static mdh_status launch_j3d7(const Plan& p, const void* const* in, void* const* out, cudaStream_t st,
                              void* hlo = nullptr, void* hhi = nullptr, bool pdl = false) {
  J7Params P;
  memset(&P, 0, sizeof(P));
  P.hlo = (float*)hlo;
  P.hhi = (float*)hhi;
  const int dz = (int)p.auxi[0], dy = (int)p.auxi[1], dx = (int)p.auxi[2], c = (int)p.auxi[3];
  const Buf& B = p.in[0];
  const Access& O = p.out[0].acc[0];
  P.u = (const float*)in[0];
  P.v = (float*)out[0];
  P.bc = B.acc[c].base;
  P.Ly = B.acc[c].L[dy];
  P.Lz = B.acc[c].L[dz];
  P.ob = O.base;
  P.oLy = O.L[dy];
  P.oLz = O.L[dz];
  P.hbase = O.base - O.L[dz];
  P.X = (int)p.size[dx];
  P.Y = (int)p.size[dy];
  P.Z = (int)p.size[dz];
  P.wc = (float)p.fparams[c];
  float* w[6] = {&P.wxm, &P.wxp, &P.wym, &P.wyp, &P.wzm, &P.wzp};
  for (int k = 0; k < 6; ++k) *w[k] = (float)p.fparams[p.auxi[4 + k]];
  int zc = p.tiles.zchunk > 0 ? p.tiles.zchunk : 64;
  if (zc > P.Z) zc = P.Z;
  P.zchunk = zc;
  const bool vin = (P.bc - 1) % 4 == 0 && P.Ly % 4 == 0 && P.Lz % 4 == 0;
  const bool vout = P.ob % 2 == 0 && P.oLy % 2 == 0 && P.oLz % 2 == 0;
  const bool vodd = P.ob % 2 == 1 && P.oLy % 2 == 0 && P.oLz % 2 == 0;
  // block: bx threads along x (4 outputs each) × 128/bx rows; tile knob per_thread = bx
  // (32 / 64 / 128).  Measured on 512³ (zchunk 8): 32 → 206.8 µs, 64 → 209.0, 128 → 219.2 —
  // the y-halo rows of a narrow, tall block are L1 hits; longer row segments do not pay
  const int bx = (p.tiles.per_thread == 64 || p.tiles.per_thread == 128) ? p.tiles.per_thread : 32;
  // x outputs per thread: 4, or 8 with tile knob vec=8 (measured 292.9 vs 208.8 µs on 512³:
  // half the threads per plane row leave too few loads in flight)
  const int nx = p.tiles.vec == 8 ? 8 : 4;
  dim3 block(bx, 128 / bx);
  dim3 grid((unsigned)((P.X + nx * bx - 1) / (nx * bx)), (unsigned)((P.Y + block.y - 1) / block.y),
            (unsigned)((P.Z + zc - 1) / zc));
  // tile knob l2pf: L2 prefetch-size hint on the vector row loads (1: 128 B, 2: 256 B).
  // Measured on 512³ (zchunk 8, 3 interleaved reps on one box): none 206.8 µs, 128 B 206.8,
  // 256 B 204.8 (5212 GB/s; 8 sweeps 1.740 -> 1.732 ms); the z+1 row loaded one step ahead
  // (software pipeline along z, +8 registers) 206.9, with the 256 B hint 206.8 — dropped
  // TMA-staged variant (tile knob stages = ring depth ≥ 3): the input must be a row-major
  // [nz][ny][nx] buffer (x stride 1, Ly = nx, Lz = ny·nx) with 16-byte aligned rows and planes
  const Buf& Bin = p.in[0];
  const int st_ring = std::min(p.tiles.stages, J7T_MAXS);
  if (st_ring >= 3 && Bin.rank == 3 && Bin.shape[2] == P.Ly && Bin.shape[1] * Bin.shape[2] == P.Lz && P.Ly % 4 == 0 &&
      P.Lz % 4 == 0 && ((uintptr_t)P.u % 16) == 0 && P.oLy > 0) {
    static PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
      void* f = nullptr;
      cudaDriverEntryPointQueryResult q;
      if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
          q == cudaDriverEntryPointSuccess)
        enc = (PFN_cuTensorMapEncodeTiled_v12000)f;
    });
    if (!enc) { set_error("cuTensorMapEncodeTiled unavailable"); return MDH_ERR_CUDA; }
    CUtensorMap map;
    cuuint64_t dims[2] = {(cuuint64_t)Bin.shape[2], (cuuint64_t)(Bin.shape[1] * Bin.shape[0])};
    cuuint64_t strides[1] = {(cuuint64_t)P.Ly * 4};
    cuuint32_t box[2] = {J7T_BX, J7T_BY};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)P.u, dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) { set_error("cuTensorMapEncodeTiled (stencil input) failed (%d)", (int)r); return MDH_ERR_CUDA; }
    // input coordinate of the centre access at the iteration origin
    const int cz = (int)(P.bc / P.Lz), cy = (int)((P.bc % P.Lz) / P.Ly), cx = (int)(P.bc % P.Ly);
    const size_t smem = (size_t)st_ring * J7T_SLOT + 1024;
    void (*tk)(CUtensorMap, J7Params, int, int, int, int, int) =
        vout ? t1_j3d7_tma_kernel<1> : (vodd ? t1_j3d7_tma_kernel<2> : t1_j3d7_tma_kernel<0>);
    static std::once_flag attr_once;
    static cudaError_t attr_err = cudaSuccess;
    std::call_once(attr_once, [] {
      for (auto k : {t1_j3d7_tma_kernel<0>, t1_j3d7_tma_kernel<1>, t1_j3d7_tma_kernel<2>}) {
        const cudaError_t e = cudaFuncSetAttribute((const void*)k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                   J7T_MAXS * J7T_SLOT + 1024);
        if (e != cudaSuccess) attr_err = e;
      }
    });
    MDH_CUDA(attr_err);
    dim3 tgrid((unsigned)((P.X + J7T_TX - 1) / J7T_TX), (unsigned)((P.Y + J7T_TY - 1) / J7T_TY),
               (unsigned)((P.Z + zc - 1) / zc));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = tgrid;
    cfg.blockDim = dim3(J7T_THREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl ? 1 : 0;
    MDH_CUDA(cudaLaunchKernelEx(&cfg, tk, map, P, st_ring, cx, cy, cz, (int)Bin.shape[1]));
    return post_launch("t1_j3d7_tma_kernel");
  }
  const int pf = p.tiles.l2pf;
  void (*kern)(J7Params) = nullptr;
#define J7(VI, VO)                                              \
  do {                                                          \
    if (nx == 8) kern = t1_j3d7_kernel<VI, VO, 8>;              \
    else if (pf == 2) kern = t1_j3d7_kernel<VI, VO, 4, 2>;      \
    else if (pf == 1) kern = t1_j3d7_kernel<VI, VO, 4, 1>;      \
    else kern = t1_j3d7_kernel<VI, VO, 4>;                      \
  } while (0)
  if (vin && vout) J7(true, 1);
  else if (vin && vodd) J7(true, 2);
  else if (vin) J7(true, 0);
  else if (vout) J7(false, 1);
  else J7(false, 0);
#undef J7
  if (pdl) {                // time-stepping: a programmatic dependent of the previous sweep
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    MDH_CUDA(cudaLaunchKernelEx(&cfg, kern, P));
  } else {
    kern<<<grid, block, 0, st>>>(P);
  }
  return post_launch("t1_j3d7_kernel");
}

// one sweep of a same-shape stencil plan with the halo stores fused into the 7-point
// kernel (mdh_stencil_sweeps, peer transport); UNSUPPORTED when the plan does not run the
// 7-point kernel or its first output plane is not buffer plane 1 (the caller then copies)
mdh_status launch_t1_halo(const Plan& p, const void* in, void* out, void* hlo, void* hhi, cudaStream_t st, bool pdl) {
  if (p.tmpl != T1_STENCIL || p.auxi.empty() || p.auxi[0] == -2) return MDH_ERR_UNSUPPORTED;
  const Access& O = p.out[0].acc[0];
  const int dz = (int)p.auxi[0];
  if (O.L[dz] <= 0 || O.base < O.L[dz] || O.base >= 2 * O.L[dz]) return MDH_ERR_UNSUPPORTED;
  const void* ins[1] = {in};
  void* outs[1] = {out};
  return launch_j3d7(p, ins, outs, st, hlo, hhi, pdl);
}

mdh_status launch_t1(const Plan& p, const void* const* in, void* const* out, void*, cudaStream_t st) {
  if (!p.auxi.empty() && p.auxi[0] == -2) return launch_box2d(p, in, out, st);
  if (!p.auxi.empty()) return launch_j3d7(p, in, out, st);
  T1Params P;
  memset(&P, 0, sizeof(P));
  // map the (up to 3) non-degenerate dims to z, y, x in dimension order (x = last)
  int dims[3] = {-1, -1, -1};
  int nd = 0;
  for (int d = 0; d < p.D; ++d)
    if (p.size[d] > 1) dims[nd++] = d;
  int dz = -1, dy = -1, dx = -1;
  if (nd >= 1) dx = dims[nd - 1];
  if (nd >= 2) dy = dims[nd - 2];
  if (nd >= 3) dz = dims[nd - 3];
  P.X = dx >= 0 ? p.size[dx] : 1;
  P.Y = dy >= 0 ? p.size[dy] : 1;
  P.Z = dz >= 0 ? p.size[dz] : 1;
  int n = 0;
  bool same_buf = true;
  for (int b = 0; b < p.n_in; ++b)
    for (int a = 0; a < p.in[b].nacc; ++a, ++n) {
      const Access& A = p.in[b].acc[a];
      P.ptr[n] = in[b];
      same_buf &= (b == 0);
      P.base[n] = A.base;
      P.Lx[n] = dx >= 0 ? A.L[dx] : 0;
      P.Ly[n] = dy >= 0 ? A.L[dy] : 0;
      P.Lz[n] = dz >= 0 ? A.L[dz] : 0;
    }
  P.nacc = n;
  P.f = p.f;
  for (int a = 0; a < n; ++a) P.w[a] = p.f == MDH_F_STENCIL ? (float)p.fparams[a] : 1.0f;
  const Access& O = p.out[0].acc[0];
  P.obase = O.base;
  P.oLx = dx >= 0 ? O.L[dx] : 0;
  P.oLy = dy >= 0 ? O.L[dy] : 0;
  P.oLz = dz >= 0 ? O.L[dz] : 0;
  P.out = out[0];
  P.odt = p.out[0].dtype;
  const int bx = 32, by = 8;
  int zc = p.tiles.zchunk > 0 ? p.tiles.zchunk : 16;
  if (P.Z < zc) zc = (int)P.Z;
  P.zchunk = zc;
  dim3 block(bx, by);
  dim3 grid((unsigned)((P.X + bx - 1) / bx), (unsigned)((P.Y + by - 1) / by), (unsigned)((P.Z + zc - 1) / zc));
  if (p.f == MDH_F_STENCIL) {
    if (n == 7 && same_buf) t1_kernel<7, MDH_F_STENCIL, true><<<grid, block, 0, st>>>(P);
    else if (n == 3 && same_buf) t1_kernel<3, MDH_F_STENCIL, true><<<grid, block, 0, st>>>(P);
    else if (same_buf) t1_kernel<0, MDH_F_STENCIL, true><<<grid, block, 0, st>>>(P);
    else t1_kernel<0, MDH_F_STENCIL, false><<<grid, block, 0, st>>>(P);
  } else if (p.f == MDH_F_MUL) {
    t1_kernel<2, MDH_F_MUL, false><<<grid, block, 0, st>>>(P);
  } else {
    t1_kernel<1, MDH_F_IDENTITY, true><<<grid, block, 0, st>>>(P);
  }
  return post_launch("t1_kernel");
}

}  // namespace mdh
