// t1_stencil.cu — T1: all-cc md_hom (no pw dims): maps and stencils (Jacobi1D/3D,
// Gaussian; Fig 3, Listing 10 caption P:308, 3-access example P:251).
//
// Every cc dim maps to the grid (A1): the innermost iteration dim to threadIdx.x (the
// contiguous dim of the buffers: 128-byte coalesced warp accesses), the next one to
// threadIdx.y, and the outermost is marched by each thread over a z-chunk so that the
// planes a stencil re-reads (z±1, y±1, x±1) are served from L1/L2 and every input
// element comes from HBM about once (A2); f = Σ_a w_a·x_a (reading C-16) in fp32
// with FMA (reading C-13).  HBM-bound: ≈8.05 B per output point for Jacobi3D.
#include <algorithm>

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

mdh_status prepare_t1(Plan* p) {
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

mdh_status launch_t1(const Plan& p, const void* const* in, void* const* out, void*, cudaStream_t st) {
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
  int zc = p.tiles.zchunk > 0 ? p.tiles.zchunk : 32;
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
