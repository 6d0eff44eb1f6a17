// t2_reduce.cu — T2: streaming reduction for pw(add|max|min) over a cheap f with
// little reuse (Dot, MatVec, row/column reductions) — SURVEY §8(a) A2-A8.
//
// HBM-bound by construction (Dot: AI 0.25 flop/B).  Design:
//   * row mode (the reduction dim is contiguous): work unit = (cc point c, split s);
//     one CTA folds a contiguous chunk of the reduction range with 128-bit
//     `ld.global.nc` loads, four independent vectors in flight per thread (A2, A4);
//     warp shuffle tree (A5) → shared memory across warps in warp order (A6);
//     with S > 1 splits, each CTA writes its partial to the workspace and the LAST
//     CTA of c (atomic ticket) folds the S partials with a fixed tree (A7) — one
//     kernel, no float atomics, bit-reproducible;
//   * column mode (the reduction dim is strided, cc contiguous): one thread per
//     (c, s) folds sequentially, coalesced across c; S > 1 uses a combine kernel.
// All T2 operators are commutative, so a strided thread mapping is allowed (C-2).
#include <algorithm>

#include "kcommon.cuh"

namespace mdh {

struct T2Params {
  const void* a;
  const void* b;
  int64_t abase, bbase, obase;
  int64_t aLr, bLr;                 // element stride along the flattened pw range
  int ncc;
  int64_t ccsize[MDH_MAX_D];        // cc dims in order (last fastest)
  int64_t aLc[MDH_MAX_D], bLc[MDH_MAX_D], oLc[MDH_MAX_D];
  int64_t Ncc, Nred, chunk;
  int S;
  void* out;
  int odt;
  void* partials;                   // V[Ncc*S]
  unsigned* tickets;                // [Ncc]
};

template <class TI> struct VecOf;
template <> struct VecOf<float> { static constexpr int W = 4; };
template <> struct VecOf<uint16_t> { static constexpr int W = 8; };
template <> struct VecOf<double> { static constexpr int W = 2; };
template <> struct VecOf<int32_t> { static constexpr int W = 4; };
template <> struct VecOf<uint32_t> { static constexpr int W = 4; };
template <> struct VecOf<long long> { static constexpr int W = 2; };

template <class TI, class V>
__device__ __forceinline__ V cvt(TI x) {
  if constexpr (std::is_same<TI, uint16_t>::value) return (V)bf16_to_f32(x);
  else return (V)x;
}

template <class TI>
__device__ __forceinline__ TI ld1(const TI* p) {
  if constexpr (std::is_same<TI, uint16_t>::value) return *p;
  else return __ldg(p);
}

__device__ __forceinline__ uint4 ld_nc_v4(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

template <class TI, class V, int OP, int F>
__device__ __forceinline__ V fold_vec(V acc, const uint4& va, const uint4& vb) {
  constexpr int W = VecOf<TI>::W;
  const TI* ea = reinterpret_cast<const TI*>(&va);
  const TI* eb = reinterpret_cast<const TI*>(&vb);
#pragma unroll
  for (int k = 0; k < W; ++k) {
    V y = (F == MDH_F_MUL) ? Arith<V>::mul(cvt<TI, V>(ea[k]), cvt<TI, V>(eb[k])) : cvt<TI, V>(ea[k]);
    acc = combine_t<OP, V>(acc, y);
  }
  return acc;
}

template <int OP, class V>
__device__ __forceinline__ V block_reduce(V v, V* sh) {
  v = warp_reduce<OP, V>(v);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  __syncthreads();
  if (lane == 0) sh[warp] = v;
  __syncthreads();
  V r = identity_t<OP, V>();
  if (warp == 0) {
    r = lane < nw ? sh[lane] : identity_t<OP, V>();
    r = warp_reduce<OP, V>(r);
  }
  return r;   // valid in thread 0
}

template <class TI, class V, int OP, int F>
__global__ void __launch_bounds__(256) t2_row_kernel(const __grid_constant__ T2Params P) {
  __shared__ V sh[32];
  __shared__ bool is_last;
  const TI* A = (const TI*)P.a;
  const TI* B = (const TI*)P.b;
  constexpr int W = VecOf<TI>::W;
  const int64_t units = P.Ncc * P.S;
  for (int64_t u = blockIdx.x; u < units; u += gridDim.x) {
    const int64_t c = u / P.S;
    const int s = (int)(u % P.S);
    int64_t ao = P.abase, bo = P.bbase, oo = P.obase, rem = c;
    for (int t = P.ncc - 1; t >= 0; --t) {
      int64_t v = rem % P.ccsize[t];
      rem /= P.ccsize[t];
      ao += P.aLc[t] * v;
      bo += P.bLc[t] * v;
      oo += P.oLc[t] * v;
    }
    const int64_t r0 = (int64_t)s * P.chunk;
    const int64_t r1 = min(P.Nred, r0 + P.chunk);
    V acc0 = identity_t<OP, V>(), acc1 = acc0, acc2 = acc0, acc3 = acc0;
    const bool unit_a = P.aLr == 1, unit_b = (F != MDH_F_MUL) || P.bLr == 1;
    int64_t r = r0;
    if (unit_a && unit_b && (F != MDH_F_MUL || ((ao - bo) % W) == 0)) {
      // scalar head up to 16-byte alignment of a (and b, same misalignment)
      int64_t mis = ((ao + r) % W + W) % W;
      int64_t head = mis ? min((int64_t)(W - mis), (int64_t)(r1 - r)) : (int64_t)0;
      for (int64_t k = threadIdx.x; k < head; k += blockDim.x) {
        V y = (F == MDH_F_MUL) ? Arith<V>::mul(cvt<TI, V>(ld1(A + ao + r + k)), cvt<TI, V>(ld1(B + bo + r + k)))
                               : cvt<TI, V>(ld1(A + ao + r + k));
        acc0 = combine_t<OP, V>(acc0, y);
      }
      r += head;
      const int64_t nvec = (r1 - r) / W;
      const uint4* va = reinterpret_cast<const uint4*>(A + ao + r);
      const uint4* vb = reinterpret_cast<const uint4*>(B + bo + r);
      const int bd = blockDim.x;
      int64_t v = threadIdx.x;
      for (; v + 3 * bd < nvec; v += 4 * bd) {
        uint4 a0 = ld_nc_v4(va + v), a1 = ld_nc_v4(va + v + bd), a2 = ld_nc_v4(va + v + 2 * bd), a3 = ld_nc_v4(va + v + 3 * bd);
        uint4 b0 = a0, b1 = a1, b2 = a2, b3 = a3;
        if (F == MDH_F_MUL) {
          b0 = ld_nc_v4(vb + v); b1 = ld_nc_v4(vb + v + bd); b2 = ld_nc_v4(vb + v + 2 * bd); b3 = ld_nc_v4(vb + v + 3 * bd);
        }
        acc0 = fold_vec<TI, V, OP, F>(acc0, a0, b0);
        acc1 = fold_vec<TI, V, OP, F>(acc1, a1, b1);
        acc2 = fold_vec<TI, V, OP, F>(acc2, a2, b2);
        acc3 = fold_vec<TI, V, OP, F>(acc3, a3, b3);
      }
      for (; v < nvec; v += bd) {
        uint4 a0 = ld_nc_v4(va + v);
        uint4 b0 = (F == MDH_F_MUL) ? ld_nc_v4(vb + v) : a0;
        acc0 = fold_vec<TI, V, OP, F>(acc0, a0, b0);
      }
      r += nvec * W;
      for (int64_t k = r + threadIdx.x; k < r1; k += blockDim.x) {
        V y = (F == MDH_F_MUL) ? Arith<V>::mul(cvt<TI, V>(ld1(A + ao + k)), cvt<TI, V>(ld1(B + bo + k)))
                               : cvt<TI, V>(ld1(A + ao + k));
        acc1 = combine_t<OP, V>(acc1, y);
      }
    } else {
      for (int64_t k = r + threadIdx.x; k < r1; k += blockDim.x) {
        V y = (F == MDH_F_MUL) ? Arith<V>::mul(cvt<TI, V>(ld1(A + ao + k * P.aLr)), cvt<TI, V>(ld1(B + bo + k * P.bLr)))
                               : cvt<TI, V>(ld1(A + ao + k * P.aLr));
        acc0 = combine_t<OP, V>(acc0, y);
      }
    }
    V acc = combine_t<OP, V>(combine_t<OP, V>(acc0, acc1), combine_t<OP, V>(acc2, acc3));
    V tot = block_reduce<OP, V>(acc, sh);
    if (P.S == 1) {
      if (threadIdx.x == 0) store_as<V>(P.out, P.odt, oo, tot);
      continue;
    }
    // two-level cross-CTA combine (A7): partial + ticket; the last CTA folds in a fixed tree
    V* part = (V*)P.partials;
    if (threadIdx.x == 0) {
      part[c * P.S + s] = tot;
      __threadfence();
      unsigned t = atomicAdd(P.tickets + c, 1u);
      is_last = (t == (unsigned)P.S - 1);
    }
    __syncthreads();
    if (is_last) {
      __threadfence();
      V x = identity_t<OP, V>();
      for (int k = threadIdx.x; k < P.S; k += blockDim.x) {
        V pv = *((volatile V*)(part + c * P.S + k));
        x = combine_t<OP, V>(x, pv);
      }
      V fin = block_reduce<OP, V>(x, sh);
      if (threadIdx.x == 0) {
        store_as<V>(P.out, P.odt, oo, fin);
        P.tickets[c] = 0u;          // self-reset for the next execute
      }
    }
    __syncthreads();
  }
}

// warp mode (S == 1, moderate contiguous rows, many cc points: MatVec): one warp per
// cc point, 128-bit loads with 4 vectors in flight per lane, shuffle tree, no smem.
template <class TI, class V, int OP, int F>
__global__ void __launch_bounds__(256) t2_warp_kernel(const __grid_constant__ T2Params P) {
  const TI* A = (const TI*)P.a;
  const TI* B = (const TI*)P.b;
  constexpr int W = VecOf<TI>::W;
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t c = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); c < P.Ncc; c += warps) {
    int64_t ao = P.abase, bo = P.bbase, oo = P.obase, rem = c;
    for (int t = P.ncc - 1; t >= 0; --t) {
      int64_t v = rem % P.ccsize[t];
      rem /= P.ccsize[t];
      ao += P.aLc[t] * v;
      bo += P.bLc[t] * v;
      oo += P.oLc[t] * v;
    }
    V acc0 = identity_t<OP, V>(), acc1 = acc0, acc2 = acc0, acc3 = acc0;
    int64_t r = 0;
    const int64_t r1 = P.Nred;
    if (F != MDH_F_MUL || ((ao - bo) % W) == 0) {
      int64_t mis = ((ao % W) + W) % W;
      int64_t head = mis ? min((int64_t)(W - mis), r1) : (int64_t)0;
      if (lane < head) {
        V y = (F == MDH_F_MUL) ? Arith<V>::mul(cvt<TI, V>(ld1(A + ao + lane)), cvt<TI, V>(ld1(B + bo + lane)))
                               : cvt<TI, V>(ld1(A + ao + lane));
        acc0 = combine_t<OP, V>(acc0, y);
      }
      r = head;
      const int64_t nvec = (r1 - r) / W;
      const uint4* va = reinterpret_cast<const uint4*>(A + ao + r);
      const uint4* vb = reinterpret_cast<const uint4*>(B + bo + r);
      int64_t v = lane;
      for (; v + 96 < nvec; v += 128) {
        uint4 a0 = ld_nc_v4(va + v), a1 = ld_nc_v4(va + v + 32), a2 = ld_nc_v4(va + v + 64), a3 = ld_nc_v4(va + v + 96);
        uint4 b0 = a0, b1 = a1, b2 = a2, b3 = a3;
        if (F == MDH_F_MUL) {
          b0 = __ldg(vb + v); b1 = __ldg(vb + v + 32); b2 = __ldg(vb + v + 64); b3 = __ldg(vb + v + 96);
        }
        acc0 = fold_vec<TI, V, OP, F>(acc0, a0, b0);
        acc1 = fold_vec<TI, V, OP, F>(acc1, a1, b1);
        acc2 = fold_vec<TI, V, OP, F>(acc2, a2, b2);
        acc3 = fold_vec<TI, V, OP, F>(acc3, a3, b3);
      }
      for (; v < nvec; v += 32) {
        uint4 a0 = ld_nc_v4(va + v);
        uint4 b0 = (F == MDH_F_MUL) ? __ldg(vb + v) : a0;
        acc0 = fold_vec<TI, V, OP, F>(acc0, a0, b0);
      }
      r += nvec * W;
    }
    for (int64_t k = r + lane; k < r1; k += 32) {
      V y = (F == MDH_F_MUL) ? Arith<V>::mul(cvt<TI, V>(ld1(A + ao + k)), cvt<TI, V>(ld1(B + bo + k)))
                             : cvt<TI, V>(ld1(A + ao + k));
      acc1 = combine_t<OP, V>(acc1, y);
    }
    V acc = combine_t<OP, V>(combine_t<OP, V>(acc0, acc1), combine_t<OP, V>(acc2, acc3));
    acc = warp_reduce<OP, V>(acc);
    if (lane == 0) store_as<V>(P.out, P.odt, oo, acc);
  }
}

// row-range mode (tile knob mode = 3; fp32 MatVec-shaped: f = MUL, the second operand the
// same vector x for every cc point, unit-stride rows of 1024·NV elements): each CTA owns a
// CONTIGUOUS range of cc points (rows), so the GPU streams ~2 rows per SM at a time through
// HBM instead of one row per resident warp (thousands of concurrent 32 KB streams), and x
// is loaded once per thread into registers (thread t holds the 16-byte chunks t + 256·j)
// instead of once per row.  The next step's rows (8/NV rows: 8 loads per thread) are
// issued before the current step's rows are folded.  Per row: thread fold in chunk order,
// warp shuffle tree, warps in order through shared memory (8 rows per barrier) — a fixed
// association, deterministic.
template <int NV, int OP>
__global__ void __launch_bounds__(256, 2) t2_rows_kernel(const __grid_constant__ T2Params P) {
  __shared__ float red[8][8];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t G = gridDim.x;
  const int64_t c0 = P.Ncc * blockIdx.x / G, c1 = P.Ncc * (blockIdx.x + 1) / G;
  const float4* xb = reinterpret_cast<const float4*>((const float*)P.b + P.bbase) + tid;
  float4 xv[NV];
#pragma unroll
  for (int j = 0; j < NV; ++j) xv[j] = __ldg(xb + 256 * j);
  auto offs = [&](int64_t c, int64_t* ao, int64_t* oo) {
    int64_t a = P.abase, o = P.obase, rem = c;
    for (int t = P.ncc - 1; t >= 0; --t) {
      const int64_t v = rem % P.ccsize[t];
      rem /= P.ccsize[t];
      a += P.aLc[t] * v;
      o += P.oLc[t] * v;
    }
    *ao = a;
    *oo = o;
  };
  auto load = [&](int64_t c, uint4* r) {
    int64_t ao, oo;
    offs(c, &ao, &oo);
    const uint4* pa = reinterpret_cast<const uint4*>((const float*)P.a + ao) + tid;
#pragma unroll
    for (int j = 0; j < NV; ++j) r[j] = ld_nc_v4(pa + 256 * j);
  };
  // R = 8 / NV rows per step, so every step has 8 16-byte loads per thread in flight
  constexpr int R = 8 / NV;
  auto load_step = [&](int64_t s, uint4* r) {
#pragma unroll
    for (int q = 0; q < R; ++q)
      if (s + q < c1) load(s + q, r + q * NV);
  };
  uint4 cur[R * NV], nxt[R * NV];
  if (c0 < c1) load_step(c0, cur);
  for (int64_t c = c0; c < c1; c += 8) {
#pragma unroll 1
    for (int qq = 0; qq < 8; qq += R) {
      const int64_t s0 = c + qq;
      if (s0 >= c1) break;                       // CTA-uniform
      if (s0 + R < c1) load_step(s0 + R, nxt);
#pragma unroll
      for (int q = 0; q < R; ++q) {
        float acc = identity_t<OP, float>();
#pragma unroll
        for (int j = 0; j < NV; ++j) {
          const float* a = reinterpret_cast<const float*>(&cur[q * NV + j]);
          acc = combine_t<OP, float>(acc, a[0] * xv[j].x);
          acc = combine_t<OP, float>(acc, a[1] * xv[j].y);
          acc = combine_t<OP, float>(acc, a[2] * xv[j].z);
          acc = combine_t<OP, float>(acc, a[3] * xv[j].w);
        }
        acc = warp_reduce<OP, float>(acc);
        if (lane == 0) red[qq + q][warp] = acc;  // rows past c1 are never read
      }
#pragma unroll
      for (int j = 0; j < R * NV; ++j) cur[j] = nxt[j];
    }
    __syncthreads();
    if (tid < 8 && c + tid < c1) {
      float s = red[tid][0];
#pragma unroll
      for (int w = 1; w < 8; ++w) s = combine_t<OP, float>(s, red[tid][w]);
      int64_t ao, oo;
      offs(c + tid, &ao, &oo);
      store_as<float>(P.out, P.odt, oo, s);
    }
    __syncthreads();
  }
}

template <class TI, class V, int OP, int F>
__global__ void __launch_bounds__(256) t2_col_kernel(const __grid_constant__ T2Params P) {
  const TI* A = (const TI*)P.a;
  const TI* B = (const TI*)P.b;
  const int64_t units = P.Ncc * P.S;
  for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < units; u += (int64_t)gridDim.x * blockDim.x) {
    const int64_t c = u % P.Ncc;
    const int64_t s = u / P.Ncc;
    int64_t ao = P.abase, bo = P.bbase, oo = P.obase, rem = c;
    for (int t = P.ncc - 1; t >= 0; --t) {
      int64_t v = rem % P.ccsize[t];
      rem /= P.ccsize[t];
      ao += P.aLc[t] * v;
      bo += P.bLc[t] * v;
      oo += P.oLc[t] * v;
    }
    const int64_t r0 = s * P.chunk, r1 = min(P.Nred, r0 + P.chunk);
    V acc = identity_t<OP, V>();
    for (int64_t k = r0; k < r1; ++k) {
      V y = (F == MDH_F_MUL) ? Arith<V>::mul(cvt<TI, V>(ld1(A + ao + k * P.aLr)), cvt<TI, V>(ld1(B + bo + k * P.bLr)))
                             : cvt<TI, V>(ld1(A + ao + k * P.aLr));
      acc = combine_t<OP, V>(acc, y);
    }
    if (P.S == 1) store_as<V>(P.out, P.odt, oo, acc);
    else ((V*)P.partials)[s * P.Ncc + c] = acc;
  }
}

template <class TI, class V, int OP>
__global__ void __launch_bounds__(256) t2_col_combine(const __grid_constant__ T2Params P) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < P.Ncc; c += (int64_t)gridDim.x * blockDim.x) {
    int64_t oo = P.obase, rem = c;
    for (int t = P.ncc - 1; t >= 0; --t) {
      int64_t v = rem % P.ccsize[t];
      rem /= P.ccsize[t];
      oo += P.oLc[t] * v;
    }
    const V* part = (const V*)P.partials;
    V acc = part[c];
    for (int s = 1; s < P.S; ++s) acc = combine_t<OP, V>(acc, part[(int64_t)s * P.Ncc + c]);
    store_as<V>(P.out, P.odt, oo, acc);
  }
}

// ------------------------------------------------------------------------- host
static bool red_linear(const Plan& p, const Access& A, int64_t* stride) {
  int last = p.red[p.nred - 1];
  int64_t L = A.L[last], mult = p.size[last];
  for (int t = p.nred - 2; t >= 0; --t) {
    int d = p.red[t];
    if (A.L[d] != L * mult) return false;
    mult *= p.size[d];
  }
  *stride = L;
  return true;
}

static int64_t compute_size(const Plan& p) {
  switch (p.compute) {
    case MDH_F64: case MDH_I64: return 8;
    default: return 4;
  }
}

mdh_status prepare_t2(Plan* p) {
  // flattened pw range must be linear in every input access (contiguous composition)
  int64_t s;
  for (int b = 0; b < p->n_in; ++b)
    if (!red_linear(*p, p->in[b].acc[0], &s)) {
      p->tmpl = T0_GENERIC;
      p->why = "pw dims not linear in the inputs: generic template";
      return prepare_t0(p);
    }
  int64_t aLr = 0;
  red_linear(*p, p->in[0].acc[0], &aLr);
  const bool row = (aLr == 1 || aLr == -1) && aLr == 1;
  const int64_t target = 148LL * 8;
  int S = 1;
  if (row) {
    int64_t min_chunk = 2048;
    int64_t smax = std::max<int64_t>(1, p->Nred / min_chunk);
    if (p->Ncc < target) S = (int)std::min<int64_t>(smax, (target + p->Ncc - 1) / p->Ncc);
  } else {
    int64_t threads = 148LL * 2048;
    if (p->Ncc < threads) S = (int)std::min<int64_t>(std::max<int64_t>(1, p->Nred / 16), (threads + p->Ncc - 1) / p->Ncc);
  }
  if (p->tiles.split > 0) S = (int)std::min<int64_t>(p->tiles.split, p->Nred);
  if (p->tiles.mode == 3 && row) S = 1;      // row-range mode: one CTA folds whole rows
  if (S < 1) S = 1;
  p->tiles.split = S;
  // 0 = column mode, 1 = row mode (CTA per unit), 2 = row mode (warp per cc point)
  p->tiles.vec = row ? ((S == 1 && p->Nred <= 65536 && p->Ncc >= 148 * 8) ? 2 : 1) : 0;
  // 3 = row-range mode (t2_rows_kernel; tile knob mode = 3): fp32 MatVec shape — f = MUL,
  // one split, unit-stride rows of 1024·{1,2,4,8} elements, the same vector for every row
  if (p->tiles.mode == 3 && row && S == 1 && p->f == MDH_F_MUL && p->n_in == 2 && p->in[0].dtype == MDH_F32 &&
      p->in[1].dtype == MDH_F32 && p->compute == MDH_F32) {
    int64_t bLr = 0;
    red_linear(*p, p->in[1].acc[0], &bLr);
    bool ok = bLr == 1 && p->Nred % 1024 == 0 && p->in[0].acc[0].base % 4 == 0 && p->in[1].acc[0].base % 4 == 0;
    const int64_t nv = p->Nred / 1024;
    ok = ok && (nv == 1 || nv == 2 || nv == 4 || nv == 8);
    for (int t = 0; ok && t < p->ncc; ++t)
      ok = p->in[1].acc[0].L[p->cc[t]] == 0 && p->in[0].acc[0].L[p->cc[t]] % 4 == 0;
    if (ok) {
      p->tiles.vec = 3;
      p->why += " (row-range MatVec kernel)";
    }
  }
  size_t part = (S > 1) ? (size_t)p->Ncc * S * compute_size(*p) : 0;
  size_t tick = (S > 1 && row) ? (size_t)p->Ncc * 4 : 0;
  p->ws_kernel = (part + 255) / 256 * 256 + (tick + 255) / 256 * 256;
  return MDH_OK;
}

template <class TI, class V>
static mdh_status launch_typed(const Plan& p, const T2Params& P, cudaStream_t st) {
  const bool row = p.tiles.vec == 1;
  const int F = p.f;
  int64_t units = P.Ncc * P.S;
  if constexpr (std::is_same<TI, float>::value) {
    // row-range mode (tile knob mode = 3): see t2_rows_kernel for the eligibility
    // (the plan checked the shape; the buffers must be 16-byte aligned, else warp mode)
    const bool ok = p.tiles.vec == 3 && ((uintptr_t)P.a & 15) == 0 && ((uintptr_t)P.b & 15) == 0;
    const int64_t nv = P.Nred / 1024;
    if (ok) {
      const int per_sm = p.tiles.per_thread >= 2 && p.tiles.per_thread <= 4 ? p.tiles.per_thread : 2;
      const unsigned g = (unsigned)std::min<int64_t>(P.Ncc, 148LL * per_sm);
#define T2_ROWS(NV)                                                                               \
  do {                                                                                            \
    if (p.redop == MDH_PW_ADD) t2_rows_kernel<NV, MDH_PW_ADD><<<g, 256, 0, st>>>(P);               \
    else if (p.redop == MDH_PW_MAX) t2_rows_kernel<NV, MDH_PW_MAX><<<g, 256, 0, st>>>(P);          \
    else t2_rows_kernel<NV, MDH_PW_MIN><<<g, 256, 0, st>>>(P);                                     \
  } while (0)
      if (nv == 1) T2_ROWS(1);
      else if (nv == 2) T2_ROWS(2);
      else if (nv == 4) T2_ROWS(4);
      else T2_ROWS(8);
#undef T2_ROWS
      return post_launch("t2_rows_kernel");
    }
  }
  if (p.tiles.vec == 2 || p.tiles.vec == 3) {
    unsigned g = (unsigned)std::min<int64_t>((P.Ncc + 7) / 8, 148LL * 16);
#define T2_WARP(OP, FF) t2_warp_kernel<TI, V, OP, FF><<<g, 256, 0, st>>>(P)
    if (F == MDH_F_MUL) {
      if (p.redop == MDH_PW_ADD) T2_WARP(MDH_PW_ADD, MDH_F_MUL);
      else if (p.redop == MDH_PW_MAX) T2_WARP(MDH_PW_MAX, MDH_F_MUL);
      else T2_WARP(MDH_PW_MIN, MDH_F_MUL);
    } else {
      if (p.redop == MDH_PW_ADD) T2_WARP(MDH_PW_ADD, MDH_F_IDENTITY);
      else if (p.redop == MDH_PW_MAX) T2_WARP(MDH_PW_MAX, MDH_F_IDENTITY);
      else T2_WARP(MDH_PW_MIN, MDH_F_IDENTITY);
    }
#undef T2_WARP
    return post_launch("t2_warp_kernel");
  }
#define T2_ROW(OP, FF) t2_row_kernel<TI, V, OP, FF><<<(unsigned)std::min<int64_t>(units, 148LL * 64), 256, 0, st>>>(P)
#define T2_COL(OP, FF) t2_col_kernel<TI, V, OP, FF><<<(unsigned)std::min<int64_t>((units + 255) / 256, 148LL * 64), 256, 0, st>>>(P)
  if (row) {
    if (F == MDH_F_MUL) {
      if (p.redop == MDH_PW_ADD) T2_ROW(MDH_PW_ADD, MDH_F_MUL);
      else if (p.redop == MDH_PW_MAX) T2_ROW(MDH_PW_MAX, MDH_F_MUL);
      else T2_ROW(MDH_PW_MIN, MDH_F_MUL);
    } else {
      if (p.redop == MDH_PW_ADD) T2_ROW(MDH_PW_ADD, MDH_F_IDENTITY);
      else if (p.redop == MDH_PW_MAX) T2_ROW(MDH_PW_MAX, MDH_F_IDENTITY);
      else T2_ROW(MDH_PW_MIN, MDH_F_IDENTITY);
    }
    return post_launch("t2_row_kernel");
  }
  if (F == MDH_F_MUL) {
    if (p.redop == MDH_PW_ADD) T2_COL(MDH_PW_ADD, MDH_F_MUL);
    else if (p.redop == MDH_PW_MAX) T2_COL(MDH_PW_MAX, MDH_F_MUL);
    else T2_COL(MDH_PW_MIN, MDH_F_MUL);
  } else {
    if (p.redop == MDH_PW_ADD) T2_COL(MDH_PW_ADD, MDH_F_IDENTITY);
    else if (p.redop == MDH_PW_MAX) T2_COL(MDH_PW_MAX, MDH_F_IDENTITY);
    else T2_COL(MDH_PW_MIN, MDH_F_IDENTITY);
  }
  MDH_TRY(post_launch("t2_col_kernel"));
  if (P.S > 1) {
    unsigned g = (unsigned)std::min<int64_t>((P.Ncc + 255) / 256, 148LL * 64);
    if (p.redop == MDH_PW_ADD) t2_col_combine<TI, V, MDH_PW_ADD><<<g, 256, 0, st>>>(P);
    else if (p.redop == MDH_PW_MAX) t2_col_combine<TI, V, MDH_PW_MAX><<<g, 256, 0, st>>>(P);
    else t2_col_combine<TI, V, MDH_PW_MIN><<<g, 256, 0, st>>>(P);
    MDH_TRY(post_launch("t2_col_combine"));
  }
#undef T2_ROW
#undef T2_COL
  return MDH_OK;
}

mdh_status launch_t2(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st) {
  T2Params P;
  memset(&P, 0, sizeof(P));
  P.a = in[0];
  P.b = p.n_in > 1 ? in[1] : in[0];
  const Access& A = p.in[0].acc[0];
  const Access& B = p.n_in > 1 ? p.in[1].acc[0] : p.in[0].acc[0];
  const Access& O = p.out[0].acc[0];
  P.abase = A.base;
  P.bbase = B.base;
  P.obase = O.base;
  red_linear(p, A, &P.aLr);
  red_linear(p, B, &P.bLr);
  P.ncc = p.ncc;
  for (int t = 0; t < p.ncc; ++t) {
    int d = p.cc[t];
    P.ccsize[t] = p.size[d];
    P.aLc[t] = A.L[d];
    P.bLc[t] = B.L[d];
    P.oLc[t] = O.L[d];
  }
  P.Ncc = p.Ncc;
  P.Nred = p.Nred;
  P.S = p.tiles.split;
  P.chunk = (p.Nred + P.S - 1) / P.S;
  P.chunk = (P.chunk + 15) / 16 * 16;
  P.out = out[0];
  P.odt = p.out[0].dtype;
  size_t part = (P.S > 1) ? (size_t)p.Ncc * P.S * compute_size(p) : 0;
  P.partials = ws;
  P.tickets = (unsigned*)((char*)ws + (part + 255) / 256 * 256);
  // the ticket words must be zero at entry: the workspace is zero-filled once by its
  // owner (mdh.h contract) and the last CTA of every cc point resets its ticket
  switch (p.in[0].dtype) {
    case MDH_F32: return launch_typed<float, float>(p, P, st);
    case MDH_BF16: return launch_typed<uint16_t, float>(p, P, st);
    case MDH_F64: return launch_typed<double, double>(p, P, st);
    case MDH_I32: return launch_typed<int32_t, int32_t>(p, P, st);
    case MDH_U32: return launch_typed<uint32_t, uint32_t>(p, P, st);
    case MDH_I64: return launch_typed<long long, long long>(p, P, st);
  }
  set_error("T2: bad dtype");
  return MDH_ERR_UNSUPPORTED;
}

}  // namespace mdh
