// t6_scan.cu — T6: the prefix-sum combine operator ps(add) (Listing 17; SURVEY
// §8(f) F1) and MBBS read as md_hom(id, (pw(add), ps(add))) (reading C-30).
//
// One ps dim d_ps is kept and folded over [0, k]; other kept (cc) dims enumerate rows c;
// pw(add) dims are folded completely.  Because every operator here is +, the result is
//   R[c, k] = Σ_{t ≤ k} z[c, t],   z[c, t] = Σ_{pw} f(x(c, t, pw))
// which the GPU evaluates as
//   K1  z[c, t]          — one thread per (c, t), sequential fold over the pw dims
//   K2  per (c, chunk)   — block inclusive scan of a 4096-element chunk (16 per thread,
//                          warp shuffles, warps in order) + the chunk total
//   K3  per row          — exclusive scan of the chunk totals (in chunk order)
//   K4  per (c, t)       — R = local scan + chunk offset, written through out_view
// (K3/K4 are skipped when a row fits one chunk).  Deterministic: fixed association order,
// no atomics.  HBM-bound: z and the local scans are each written and read once.
#include <algorithm>

#include "kcommon.cuh"

namespace mdh {

constexpr int T6_CHUNK = 4096, T6_THREADS = 256, T6_PER = T6_CHUNK / T6_THREADS;

struct T6Params {
  const void* ptr[2];
  int dt[2];
  int nacc, f;
  int64_t base[2];
  int64_t Lrow[2][MDH_MAX_D];        // input strides of the row (other kept) dims
  int64_t Lt[2];                     // input stride of the ps dim
  int nrowd;
  int64_t rowsize[MDH_MAX_D];
  int64_t orowL[MDH_MAX_D], oLt, obase;
  int npw;
  int64_t pwsize[MDH_MAX_D], Lpw[2][MDH_MAX_D];
  int64_t Nc, T, nq;
  int direct;                        // no pw dims, f = IDENTITY: the scan reads x itself
  void* out;
  int odt;
  void* z;        // V[Nc][T]
  void* loc;      // V[Nc][T]
  void* sums;     // V[Nc][nq]
};

// K1 with the pw range split over threadIdx.y (8 contiguous sub-ranges, folded in order
// through shared memory): 32 consecutive (c, t) points per block row keep loads coalesced
template <class V>
__global__ void __launch_bounds__(256) t6_fold_kernel(const __grid_constant__ T6Params P) {
  __shared__ V part[8][32];
  const int64_t total = P.Nc * P.T;
  int64_t npts = 1;
  for (int q = 0; q < P.npw; ++q) npts *= P.pwsize[q];
  const int64_t per = (npts + 7) / 8;
  for (int64_t eb = (int64_t)blockIdx.x * 32; eb < total; eb += (int64_t)gridDim.x * 32) {
    const int64_t e = eb + threadIdx.x;
    const int64_t r0 = min(npts, (int64_t)threadIdx.y * per), r1 = min(npts, r0 + per);
    V acc = (V)0;
    if (e < total && r0 < r1) {
    const int64_t c = e / P.T, t = e % P.T;
    int64_t off[2] = {P.base[0] + P.Lt[0] * t, P.base[1] + P.Lt[1] * t};
    int64_t rem = c;
    for (int q = P.nrowd - 1; q >= 0; --q) {
      const int64_t v = rem % P.rowsize[q];
      rem /= P.rowsize[q];
      off[0] += P.Lrow[0][q] * v;
      off[1] += P.Lrow[1][q] * v;
    }
    int64_t idx[MDH_MAX_D];
    int64_t rr = r0;
    for (int q = P.npw - 1; q >= 0; --q) {      // odometer start = r0 (mixed radix)
      idx[q] = rr % P.pwsize[q];
      rr /= P.pwsize[q];
      off[0] += P.Lpw[0][q] * idx[q];
      off[1] += P.Lpw[1][q] * idx[q];
    }
    for (int64_t r = r0; r < r1; ++r) {
      const V x0 = load_as<V>(P.ptr[0], P.dt[0], off[0]);
      const V y = (P.f == MDH_F_MUL) ? Arith<V>::mul(x0, load_as<V>(P.ptr[1], P.dt[1], off[1])) : x0;
      acc = (r == r0) ? y : Arith<V>::add(acc, y);
      for (int q = P.npw - 1; q >= 0; --q) {
        if (++idx[q] < P.pwsize[q]) { off[0] += P.Lpw[0][q]; off[1] += P.Lpw[1][q]; break; }
        off[0] -= P.Lpw[0][q] * (P.pwsize[q] - 1);
        off[1] -= P.Lpw[1][q] * (P.pwsize[q] - 1);
        idx[q] = 0;
      }
    }
    }
    part[threadIdx.y][threadIdx.x] = acc;
    __syncthreads();
    if (threadIdx.y == 0 && e < total) {
      V s = part[0][threadIdx.x];
      for (int y = 1; y < 8; ++y) s = Arith<V>::add(s, part[y][threadIdx.x]);   // sub-range order
      ((V*)P.z)[e] = s;
    }
    __syncthreads();
  }
}

__device__ __forceinline__ int64_t t6_out_offset(const T6Params& P, int64_t c, int64_t t) {
  int64_t o = P.obase + P.oLt * t, rem = c;
  for (int q = P.nrowd - 1; q >= 0; --q) {
    const int64_t v = rem % P.rowsize[q];
    rem /= P.rowsize[q];
    o += P.orowL[q] * v;
  }
  return o;
}

// block inclusive scan of one chunk; writes either the final output (single chunk) or the
// local scan + the chunk total
template <class V>
__global__ void __launch_bounds__(T6_THREADS) t6_chunk_scan_kernel(const __grid_constant__ T6Params P) {
  __shared__ V wsum[T6_THREADS / 32];
  __shared__ V tile[T6_CHUNK + T6_CHUNK / 32];      // padded: thread k reads 16 consecutive
  const int64_t c = blockIdx.y, q = blockIdx.x;
  const int64_t tb = q * T6_CHUNK;
  const int64_t t0 = tb + (int64_t)threadIdx.x * T6_PER;
  const V* zr = (const V*)P.z + c * P.T;
  // no pw dims and f = IDENTITY: scan the input directly (K1 skipped)
  int64_t xrow = P.base[0];
  if (P.direct) {
    int64_t rem = c;
    for (int d = P.nrowd - 1; d >= 0; --d) {
      const int64_t v = rem % P.rowsize[d];
      rem /= P.rowsize[d];
      xrow += P.Lrow[0][d] * v;
    }
  }
  // coalesced staging of the chunk (consecutive threads, consecutive elements)
#pragma unroll
  for (int k = 0; k < T6_PER; ++k) {
    const int j = k * T6_THREADS + threadIdx.x;
    const int64_t t = tb + j;
    tile[j + (j >> 5)] = t < P.T ? (P.direct ? load_as<V>(P.ptr[0], P.dt[0], xrow + P.Lt[0] * t) : zr[t]) : (V)0;
  }
  __syncthreads();
  V v[T6_PER];
  V run = (V)0;
#pragma unroll
  for (int k = 0; k < T6_PER; ++k) {
    const int j = threadIdx.x * T6_PER + k;
    const V x = tile[j + (j >> 5)];
    run = k == 0 ? x : Arith<V>::add(run, x);
    v[k] = run;
  }
  // exclusive prefix of the thread totals: warp shuffle scan, then warps in order
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  V incl = run;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const V n = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl = Arith<V>::add(n, incl);
  }
  if (lane == 31) wsum[warp] = incl;
  __syncthreads();
  V base = (V)0;
  for (int w = 0; w < warp; ++w) base = Arith<V>::add(base, wsum[w]);
  const V prev = __shfl_up_sync(0xffffffffu, incl, 1);     // inclusive total of lane-1
  const V excl = lane == 0 ? base : Arith<V>::add(base, prev);
  const bool single = P.nq == 1;
  __syncthreads();
#pragma unroll
  for (int k = 0; k < T6_PER; ++k) {
    const int j = threadIdx.x * T6_PER + k;
    tile[j + (j >> 5)] = (threadIdx.x == 0 && warp == 0) ? v[k] : Arith<V>::add(excl, v[k]);
  }
  __syncthreads();
  // coalesced write-back
#pragma unroll
  for (int k = 0; k < T6_PER; ++k) {
    const int j = k * T6_THREADS + threadIdx.x;
    const int64_t t = tb + j;
    if (t >= P.T) break;
    const V r = tile[j + (j >> 5)];
    if (single) store_as<V>(P.out, P.odt, t6_out_offset(P, c, t), r);
    else ((V*)P.loc)[c * P.T + t] = r;
  }
  if (!single && threadIdx.x == T6_THREADS - 1) ((V*)P.sums)[c * P.nq + q] = Arith<V>::add(excl, run);
}

// exclusive scan of each row's chunk totals, in chunk order: one CTA per row, tiles of
// 256 totals scanned with warp shuffles and a running carry (fixed association order)
template <class V>
__global__ void __launch_bounds__(256) t6_sums_kernel(const __grid_constant__ T6Params P) {
  __shared__ V wsum[8];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int64_t c = blockIdx.x; c < P.Nc; c += gridDim.x) {
    V* s = (V*)P.sums + c * P.nq;
    V carry = (V)0;
    for (int64_t q0 = 0; q0 < P.nq; q0 += 256) {
      const int64_t q = q0 + threadIdx.x;
      const V x = q < P.nq ? s[q] : (V)0;
      V incl = x;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const V n = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl = Arith<V>::add(n, incl);
      }
      __syncthreads();
      if (lane == 31) wsum[warp] = incl;
      __syncthreads();
      V base = carry;
      for (int w = 0; w < warp; ++w) base = Arith<V>::add(base, wsum[w]);
      const V prev = __shfl_up_sync(0xffffffffu, incl, 1);
      const V excl = lane == 0 ? base : Arith<V>::add(base, prev);
      if (q < P.nq) s[q] = excl;
      V tot = carry;
      for (int w = 0; w < 8; ++w) tot = Arith<V>::add(tot, wsum[w]);
      carry = tot;
    }
  }
}

template <class V>
__global__ void __launch_bounds__(256) t6_fix_kernel(const __grid_constant__ T6Params P) {
  const int64_t total = P.Nc * P.T;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t c = e / P.T, t = e % P.T, q = t / T6_CHUNK;
    const V l = ((const V*)P.loc)[e];
    const V r = q == 0 ? l : Arith<V>::add(((const V*)P.sums)[c * P.nq + q], l);
    store_as<V>(P.out, P.odt, t6_out_offset(P, c, t), r);
  }
}

// --------------------------------------------------------------------------- host
static int64_t vsize(mdh_dtype t) { return (t == MDH_F64 || t == MDH_I64) ? 8 : 4; }

mdh_status prepare_t6(Plan* p) {
  int nout_acc = 0;
  for (int b = 0; b < p->n_out; ++b) nout_acc += p->out[b].nacc;
  const bool ok = p->nps == 1 && (p->f == MDH_F_IDENTITY || p->f == MDH_F_MUL) && p->n_in_acc <= 2 && nout_acc == 1 &&
                  p->compute != MDH_BF16;
  if (!ok) {
    p->tmpl = T0_GENERIC;
    p->why = "ps outside the scan fast path: generic template";
    return prepare_t0(p);
  }
  const int64_t T = p->size[p->ps[0]];
  const int64_t Nc = p->Ncc / T;
  const int64_t nq = (T + T6_CHUNK - 1) / T6_CHUNK;
  const int64_t vs = vsize(p->compute);
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  p->ws_kernel = al((size_t)Nc * T * vs) + (nq > 1 ? al((size_t)Nc * T * vs) + al((size_t)Nc * nq * vs) : 0);
  return MDH_OK;
}

template <class V>
static mdh_status launch_typed(const T6Params& P, cudaStream_t st) {
  const int64_t total = P.Nc * P.T;
  const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>((total + 255) / 256, 148LL * 32));
  if (!P.direct) {
    const unsigned gf = (unsigned)std::max<int64_t>(1, std::min<int64_t>((total + 31) / 32, 148LL * 64));
    t6_fold_kernel<V><<<gf, dim3(32, 8), 0, st>>>(P);
    MDH_TRY(post_launch("t6_fold_kernel"));
  }
  if (P.Nc > 65535) { set_error("T6: too many rows"); return MDH_ERR_UNSUPPORTED; }
  dim3 grid((unsigned)P.nq, (unsigned)P.Nc);
  t6_chunk_scan_kernel<V><<<grid, T6_THREADS, 0, st>>>(P);
  MDH_TRY(post_launch("t6_chunk_scan_kernel"));
  if (P.nq > 1) {
    t6_sums_kernel<V><<<(unsigned)std::min<int64_t>(P.Nc, 148LL * 8), 256, 0, st>>>(P);
    MDH_TRY(post_launch("t6_sums_kernel"));
    t6_fix_kernel<V><<<g, 256, 0, st>>>(P);
    MDH_TRY(post_launch("t6_fix_kernel"));
  }
  return MDH_OK;
}

mdh_status launch_t6(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st) {
  T6Params P;
  memset(&P, 0, sizeof(P));
  const int dps = p.ps[0];
  int n = 0;
  for (int b = 0; b < p.n_in; ++b)
    for (int a = 0; a < p.in[b].nacc; ++a, ++n) {
      P.ptr[n] = in[b];
      P.dt[n] = p.in[b].dtype;
      P.base[n] = p.in[b].acc[a].base;
    }
  P.nacc = n;
  if (n == 1) { P.ptr[1] = P.ptr[0]; P.dt[1] = P.dt[0]; P.base[1] = P.base[0]; }
  P.f = p.f;
  const Access* A[2] = {nullptr, nullptr};
  n = 0;
  for (int b = 0; b < p.n_in; ++b)
    for (int a = 0; a < p.in[b].nacc; ++a) A[n++] = &p.in[b].acc[a];
  if (!A[1]) A[1] = A[0];
  const Access& O = p.out[0].acc[0];
  P.Lt[0] = A[0]->L[dps];
  P.Lt[1] = A[1]->L[dps];
  P.oLt = O.L[dps];
  P.obase = O.base;
  for (int t = 0; t < p.ncc; ++t) {
    const int d = p.cc[t];
    if (d == dps) continue;
    P.rowsize[P.nrowd] = p.size[d];
    P.Lrow[0][P.nrowd] = A[0]->L[d];
    P.Lrow[1][P.nrowd] = A[1]->L[d];
    P.orowL[P.nrowd] = O.L[d];
    ++P.nrowd;
  }
  for (int t = 0; t < p.nred; ++t) {
    const int d = p.red[t];
    if (d == dps) continue;
    P.pwsize[P.npw] = p.size[d];
    P.Lpw[0][P.npw] = A[0]->L[d];
    P.Lpw[1][P.npw] = A[1]->L[d];
    ++P.npw;
  }
  P.T = p.size[dps];
  P.Nc = p.Ncc / P.T;
  P.direct = P.npw == 0 && P.f == MDH_F_IDENTITY;
  P.nq = (P.T + T6_CHUNK - 1) / T6_CHUNK;
  P.out = out[0];
  P.odt = p.out[0].dtype;
  const int64_t vs = vsize(p.compute);
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  char* w = (char*)ws;
  P.z = w;
  P.loc = w + al((size_t)P.Nc * P.T * vs);
  P.sums = (char*)P.loc + al((size_t)P.Nc * P.T * vs);
  switch (p.compute) {
    case MDH_F32: return launch_typed<float>(P, st);
    case MDH_F64: return launch_typed<double>(P, st);
    case MDH_I32: return launch_typed<int32_t>(P, st);
    case MDH_U32: return launch_typed<uint32_t>(P, st);
    case MDH_I64: return launch_typed<long long>(P, st);
    default: set_error("T6: unsupported type"); return MDH_ERR_UNSUPPORTED;
  }
}

}  // namespace mdh
