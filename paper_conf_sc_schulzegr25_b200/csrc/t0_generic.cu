// t0_generic.cu — T0: the catch-all GPU template.  One thread per cc point evaluates
// the md_hom definition (fn.2) directly: gather every input access through
// its affine index function (inp_view), apply f, left-fold the pw dims
// in lexicographic order (Listing 16; reading C-1), write through out_view.
// Used for specs no specialised template covers (e.g. strided custom outputs); it is
// never the path of a benchmarked config.
#include "kcommon.cuh"
#include "prl_common.cuh"

namespace mdh {

constexpr int T0_MAX_ACC = 24;

struct T0Params {
  int D, ncc, nred, op, f, nacc, nout, nps;
  int kind[MDH_MAX_D];                // per dim: 0 cc, 1 pw, 2 ps (kept and folded over [0,k])
  int64_t size[MDH_MAX_D];
  int cc[MDH_MAX_D], red[MDH_MAX_D];
  int64_t Ncc, Nred;
  const void* ptr[T0_MAX_ACC];
  int dt[T0_MAX_ACC];
  int64_t base[T0_MAX_ACC];
  int64_t L[T0_MAX_ACC][MDH_MAX_D];
  double w[T0_MAX_ACC];
  void* optr[3];
  int odt[3];
  int64_t obase[3];
  int64_t oL[3][MDH_MAX_D];
};

template <class V>
__global__ void __launch_bounds__(128) t0_kernel(const __grid_constant__ T0Params P) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < P.Ncc;
       c += (int64_t)gridDim.x * blockDim.x) {
    int64_t off[T0_MAX_ACC];
    for (int a = 0; a < P.nacc; ++a) off[a] = P.base[a];
    int64_t ooff = P.obase[0];
    int64_t rem = c;
    int64_t lim[MDH_MAX_D];            // fold extent per dim: I_d (pw) or k+1 (ps)
    for (int d = 0; d < P.D; ++d) lim[d] = P.size[d];
    for (int t = P.ncc - 1; t >= 0; --t) {
      int d = P.cc[t];
      int64_t v = rem % P.size[d];
      rem /= P.size[d];
      if (P.kind[d] == 2) lim[d] = v + 1;              // ps: inputs are folded from index 0
      else for (int a = 0; a < P.nacc; ++a) off[a] += P.L[a][d] * v;
      ooff += P.oL[0][d] * v;
    }
    int64_t ridx[MDH_MAX_D];
    for (int t = 0; t < P.nred; ++t) ridx[t] = 0;
    V acc = (V)0;
    int64_t nred_here = 1;
    for (int t = 0; t < P.nred; ++t) nred_here *= lim[P.red[t]];
    for (int64_t r = 0; r < nred_here; ++r) {
      V y;
      if (P.f == MDH_F_STENCIL) {
        y = (V)P.w[0] * load_as<V>(P.ptr[0], P.dt[0], off[0]);
        for (int a = 1; a < P.nacc; ++a) y = Arith<V>::mul_add(y, (V)P.w[a], load_as<V>(P.ptr[a], P.dt[a], off[a]));
      } else if (P.f == MDH_F_MUL) {
        y = Arith<V>::mul(load_as<V>(P.ptr[0], P.dt[0], off[0]), load_as<V>(P.ptr[1], P.dt[1], off[1]));
      } else {
        y = load_as<V>(P.ptr[0], P.dt[0], off[0]);
      }
      acc = (r == 0) ? y : combine_op<V>(P.op, acc, y);    // left fold, lhs = lower range
      // odometer over the folded dims (last fastest = lexicographic order)
      for (int t = P.nred - 1; t >= 0; --t) {
        int d = P.red[t];
        if (++ridx[t] < lim[d]) {
          for (int a = 0; a < P.nacc; ++a) off[a] += P.L[a][d];
          break;
        }
        for (int a = 0; a < P.nacc; ++a) off[a] -= P.L[a][d] * (lim[d] - 1);
        ridx[t] = 0;
      }
    }
    store_as<V>(P.optr[0], P.odt[0], ooff, acc);
  }
}

__global__ void __launch_bounds__(128) t0_prl_kernel(const __grid_constant__ T0Params P) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < P.Ncc;
       c += (int64_t)gridDim.x * blockDim.x) {
    int64_t off[17], oo[3];
    for (int a = 0; a < 17; ++a) off[a] = P.base[a];
    for (int b = 0; b < 3; ++b) oo[b] = P.obase[b];
    int64_t rem = c;
    for (int t = P.ncc - 1; t >= 0; --t) {
      int d = P.cc[t];
      int64_t v = rem % P.size[d];
      rem /= P.size[d];
      for (int a = 0; a < 17; ++a) off[a] += P.L[a][d] * v;
      for (int b = 0; b < 3; ++b) oo[b] += P.oL[b][d] * v;
    }
    int64_t ridx[MDH_MAX_D];
    for (int t = 0; t < P.nred; ++t) ridx[t] = 0;
    PrlRec acc;
    for (int64_t r = 0; r < P.Nred; ++r) {
      uint32_t mask = 0;
      for (int k = 0; k < 8; ++k)
        mask |= (((const uint32_t*)P.ptr[k])[off[k]] == ((const uint32_t*)P.ptr[8 + k])[off[8 + k]] ? 1u : 0u) << k;
      PrlRec y;
      y.id = ((const long long*)P.ptr[16])[off[16]];
      double wgt = 0.0;
      for (int k = 0; k < 8; ++k) wgt = __dadd_rn(wgt, ((mask >> k) & 1u) ? P.w[k] : P.w[8 + k]);
      y.w = wgt;
      y.m = mask == 0xFFu ? 14 : __popc(mask);
      acc = (r == 0) ? y : prl_combine(P.op, acc, y);
      for (int t = P.nred - 1; t >= 0; --t) {
        int d = P.red[t];
        if (++ridx[t] < P.size[d]) {
          for (int a = 0; a < 17; ++a) off[a] += P.L[a][d];
          break;
        }
        for (int a = 0; a < 17; ++a) off[a] -= P.L[a][d] * (P.size[d] - 1);
        ridx[t] = 0;
      }
    }
    ((long long*)P.optr[0])[oo[0]] = acc.id;
    ((double*)P.optr[1])[oo[1]] = acc.w;
    ((int32_t*)P.optr[2])[oo[2]] = acc.m;
  }
}

mdh_status prepare_t0(Plan* p) {
  if (p->n_in_acc > T0_MAX_ACC) {
    set_error("the generic template handles at most %d input accesses", T0_MAX_ACC);
    return MDH_ERR_UNSUPPORTED;
  }
  int nout_acc = 0;
  for (int b = 0; b < p->n_out; ++b) nout_acc += p->out[b].nacc;
  if (nout_acc > 3 || (p->f != MDH_F_PRL_COMPARE && nout_acc != 1)) {
    set_error("the generic template writes one output access per point (three for PRL)");
    return MDH_ERR_UNSUPPORTED;
  }
  p->ws_kernel = 0;
  return MDH_OK;
}

mdh_status launch_t0(const Plan& p, const void* const* in, void* const* out, void*, cudaStream_t st) {
  T0Params P;
  memset(&P, 0, sizeof(P));
  P.D = p.D;
  P.ncc = p.ncc;
  P.nred = p.nred;
  P.nps = p.nps;
  for (int d = 0; d < MDH_MAX_D; ++d)
    P.kind[d] = d >= p.D ? 0 : (p.op[d] == MDH_CC ? 0 : (p.op[d] == MDH_PS_ADD ? 2 : 1));
  P.op = p.redop;
  P.f = p.f;
  P.Ncc = p.Ncc;
  P.Nred = p.Nred;
  for (int d = 0; d < MDH_MAX_D; ++d) {
    P.size[d] = p.size[d];
    P.cc[d] = p.cc[d];
    P.red[d] = p.red[d];
  }
  int n = 0;
  for (int b = 0; b < p.n_in; ++b)
    for (int a = 0; a < p.in[b].nacc; ++a, ++n) {
      P.ptr[n] = in[b];
      P.dt[n] = p.in[b].dtype;
      P.base[n] = p.in[b].acc[a].base;
      for (int d = 0; d < MDH_MAX_D; ++d) P.L[n][d] = p.in[b].acc[a].L[d];
    }
  P.nacc = n;
  for (size_t k = 0; k < p.fparams.size() && k < (size_t)T0_MAX_ACC; ++k) P.w[k] = p.fparams[k];
  int o = 0;
  for (int b = 0; b < p.n_out; ++b)
    for (int a = 0; a < p.out[b].nacc; ++a, ++o) {
      P.optr[o] = out[b];
      P.odt[o] = p.out[b].dtype;
      P.obase[o] = p.out[b].acc[a].base;
      for (int d = 0; d < MDH_MAX_D; ++d) P.oL[o][d] = p.out[b].acc[a].L[d];
    }
  P.nout = o;
  int64_t blocks = (p.Ncc + 127) / 128;
  if (blocks > 148 * 64) blocks = 148 * 64;
  dim3 grid((unsigned)blocks);
  if (p.f == MDH_F_PRL_COMPARE) {
    t0_prl_kernel<<<grid, 128, 0, st>>>(P);
  } else {
    switch (p.compute) {
      case MDH_F32: t0_kernel<float><<<grid, 128, 0, st>>>(P); break;
      case MDH_F64: t0_kernel<double><<<grid, 128, 0, st>>>(P); break;
      case MDH_I32: t0_kernel<int32_t><<<grid, 128, 0, st>>>(P); break;
      case MDH_U32: t0_kernel<uint32_t><<<grid, 128, 0, st>>>(P); break;
      case MDH_I64: t0_kernel<long long><<<grid, 128, 0, st>>>(P); break;
      default: set_error("T0: unsupported compute type"); return MDH_ERR_UNSUPPORTED;
    }
  }
  return post_launch("t0_kernel");
}

}  // namespace mdh
