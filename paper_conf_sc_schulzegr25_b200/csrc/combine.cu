// combine.cu — the ordered ⊗-fold of S partial results (K-combine):
//   out[ω(j)] = p_0[ω(j)] ⊗ p_1[ω(j)] ⊗ … ⊗ p_{S-1}[ω(j)]   for every cc point j,
// lhs = lower index range (Listing 16 applied S-1 times; reading C-2), so it also
// serves the non-commutative PRL rule.  Used by mdh_combine_partials (virtual shards,
// homomorphism tests) and after the allgather of a pw-dim shard.
// Elements outside the image of ω are untouched (reading C-5).
#include <algorithm>

#include "kcommon.cuh"
#include "prl_common.cuh"

namespace mdh {

constexpr int CMB_MAX = 96;   // S * n_out pointers

struct CmbParams {
  const void* part[CMB_MAX];
  void* out[3];
  int dt[3];
  int S, nout, op, prl;
  int ncc;
  int64_t ccsize[MDH_MAX_D];
  int64_t oL[3][MDH_MAX_D];
  int64_t obase[3];
  int64_t Ncc;
};

template <class V>
__global__ void __launch_bounds__(256) combine_kernel(const __grid_constant__ CmbParams P) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < P.Ncc; j += (int64_t)gridDim.x * blockDim.x) {
    int64_t o[3] = {P.obase[0], P.obase[1], P.obase[2]};
    int64_t rem = j;
    for (int t = P.ncc - 1; t >= 0; --t) {
      int64_t v = rem % P.ccsize[t];
      rem /= P.ccsize[t];
      for (int b = 0; b < P.nout; ++b) o[b] += P.oL[b][t] * v;
    }
    if (P.prl) {
      PrlRec acc{((const long long*)P.part[0])[o[0]], ((const double*)P.part[1])[o[1]], ((const int32_t*)P.part[2])[o[2]]};
      for (int s = 1; s < P.S; ++s) {
        PrlRec r{((const long long*)P.part[s * 3 + 0])[o[0]], ((const double*)P.part[s * 3 + 1])[o[1]],
                 ((const int32_t*)P.part[s * 3 + 2])[o[2]]};
        acc = prl_combine(P.op, acc, r);
      }
      ((long long*)P.out[0])[o[0]] = acc.id;
      ((double*)P.out[1])[o[1]] = acc.w;
      ((int32_t*)P.out[2])[o[2]] = acc.m;
    } else {
      V acc = load_as<V>(P.part[0], P.dt[0], o[0]);
      for (int s = 1; s < P.S; ++s) acc = combine_op<V>(P.op, acc, load_as<V>(P.part[s], P.dt[0], o[0]));
      store_as<V>(P.out[0], P.dt[0], o[0], acc);
    }
  }
}

mdh_status launch_combine(const Plan& p, const void* const* partials, int S, void* const* out, cudaStream_t st) {
  const bool prl = p.f == MDH_F_PRL_COMPARE;
  int nout_acc = 0;
  for (int b = 0; b < p.n_out; ++b) nout_acc += p.out[b].nacc;
  if (nout_acc != p.n_out || (!prl && p.n_out != 1) || S * p.n_out > CMB_MAX) {
    set_error("combine: at most %d partial buffers with one access per output", CMB_MAX);
    return MDH_ERR_UNSUPPORTED;
  }
  CmbParams P;
  memset(&P, 0, sizeof(P));
  for (int k = 0; k < S * p.n_out; ++k) P.part[k] = partials[k];
  for (int b = 0; b < p.n_out; ++b) {
    P.out[b] = out[b];
    P.dt[b] = p.out[b].dtype;
    P.obase[b] = p.out[b].acc[0].base;
    for (int t = 0; t < p.ncc; ++t) P.oL[b][t] = p.out[b].acc[0].L[p.cc[t]];
  }
  P.S = S;
  P.nout = p.n_out;
  P.op = p.redop;
  P.prl = prl;
  P.ncc = p.ncc;
  for (int t = 0; t < p.ncc; ++t) P.ccsize[t] = p.size[p.cc[t]];
  P.Ncc = p.Ncc;
  unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>((p.Ncc + 255) / 256, 148 * 16));
  mdh_dtype t = prl ? MDH_F64 : p.compute;
  switch (t) {
    case MDH_F32: combine_kernel<float><<<g, 256, 0, st>>>(P); break;
    case MDH_F64: combine_kernel<double><<<g, 256, 0, st>>>(P); break;
    case MDH_I32: combine_kernel<int32_t><<<g, 256, 0, st>>>(P); break;
    case MDH_U32: combine_kernel<uint32_t><<<g, 256, 0, st>>>(P); break;
    case MDH_I64: combine_kernel<long long><<<g, 256, 0, st>>>(P); break;
    default: set_error("combine: bad type"); return MDH_ERR_UNSUPPORTED;
  }
  return post_launch("combine_kernel");
}

}  // namespace mdh
