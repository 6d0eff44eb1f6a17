// t5_prl.cu — T5: probabilistic record linkage (Listing 11; Fig 3):
// md_hom[N,I](PRL_COMPARE, (cc, pw(prl)))  — every new record n is compared with every
// DB record i and the comparison records are folded with the custom pw operator.
//
// ALU-bound (≈2^34 pair evaluations at the config, ~40 MB of data): each thread keeps
// R new records in registers; the CTA stages DB tiles (8 u32 fields + id) in shared
// memory and every thread folds its R records over the tile in ascending i (A4, the
// order-preserving mapping required by the non-commutative paper rule, reading C-2).
// f (reading C-18): an 8-bit agreement mask from 8 u32 equality tests; the fold only
// needs the ORDER of (id==14, weight) which the plan precomputes per mask as a dense
// rank (ties equal), so a pair costs the 8 compares, one conflict-free byte lookup
// (the rank table is replicated per lane/bank) and a lexicographic compare with the
// running best (rank, match_id).  The fp64 weight Σ_k (bit_k ? wa_k : wd_k), summed in
// field order, and id_measure are produced only for the final best record.
// The reduction dim is split over CTAs when N alone cannot fill the GPU (orientation
// B, 2^14 × 2^20; reading C-20): partial records [S][N] are folded in split order by
// a combine kernel (A7), lhs = lower range.
#include <algorithm>
#include <vector>

#include "kcommon.cuh"
#include "prl_common.cuh"

namespace mdh {

constexpr int T5_THREADS = 256;
constexpr int T5_R = 4;           // new records per thread
constexpr int T5_TILE = 512;      // DB records per smem tile

struct T5Params {
  const uint32_t* nf[8];
  const uint32_t* df[8];
  const long long* dbid;
  int64_t nbase[8], nL[8];        // new field k of record n at nbase + nL*n
  int64_t dbase[9], dL[9];        // db field k (k=8: id) of record i at dbase + dL*i
  int64_t N, I, ichunk;
  int S, op;
  const uint8_t* rank32;          // [64][32] words: byte (mask&3) of word (mask>>2)*32+lane
  const double* wtab;             // [256] fp64 weights
  // outputs: final (through ω) or partials [S][N]
  long long* oid;
  double* ow;
  int32_t* om;
  int64_t obase[3], oL[3];
  long long* pid;
  double* pw;
  int32_t* pm;
};

__global__ void __launch_bounds__(T5_THREADS) t5_kernel(const __grid_constant__ T5Params P) {
  __shared__ __align__(16) uint32_t sf[T5_TILE][8];
  __shared__ long long sid[T5_TILE];
  __shared__ uint32_t srank[64 * 32];
  const int tid = threadIdx.x, lane = tid & 31;
  for (int k = tid; k < 64 * 32; k += T5_THREADS) srank[k] = ((const uint32_t*)P.rank32)[k];
  const int64_t nblk = (P.N + T5_THREADS * T5_R - 1) / (T5_THREADS * T5_R);
  const int64_t bn = blockIdx.x % nblk;
  const int s = (int)(blockIdx.x / nblk);
  const int64_t i0 = (int64_t)s * P.ichunk;
  const int64_t i1 = min(P.I, i0 + P.ichunk);
  uint32_t nv[T5_R][8];
  int64_t nn[T5_R];
  bool valid[T5_R];
#pragma unroll
  for (int r = 0; r < T5_R; ++r) {
    nn[r] = bn * (T5_THREADS * T5_R) + r * T5_THREADS + tid;
    valid[r] = nn[r] < P.N;
#pragma unroll
    for (int k = 0; k < 8; ++k) nv[r][k] = valid[r] ? __ldg(P.nf[k] + P.nbase[k] + P.nL[k] * nn[r]) : 0xFFFFFFFFu;
  }
  int brank[T5_R];
  long long bid[T5_R];
  uint32_t bmask[T5_R];
  bool b14[T5_R];
#pragma unroll
  for (int r = 0; r < T5_R; ++r) { brank[r] = -1; bid[r] = 0; bmask[r] = 0; b14[r] = false; }
  const bool paper = P.op == MDH_PW_PRL_PAPER;
  for (int64_t t0 = i0; t0 < i1; t0 += T5_TILE) {
    const int cnt = (int)min((int64_t)T5_TILE, (int64_t)(i1 - t0));
    __syncthreads();
    for (int j = tid; j < cnt; j += T5_THREADS) {
      const int64_t i = t0 + j;
#pragma unroll
      for (int k = 0; k < 8; ++k) sf[j][k] = __ldg(P.df[k] + P.dbase[k] + P.dL[k] * i);
      sid[j] = __ldg(P.dbid + P.dbase[8] + P.dL[8] * i);
    }
    __syncthreads();
    for (int j = 0; j < cnt; ++j) {
      const uint4 lo = *reinterpret_cast<const uint4*>(&sf[j][0]);
      const uint4 hi = *reinterpret_cast<const uint4*>(&sf[j][4]);
      const long long id = sid[j];
#pragma unroll
      for (int r = 0; r < T5_R; ++r) {
        uint32_t m = (uint32_t)(nv[r][0] == lo.x) | ((uint32_t)(nv[r][1] == lo.y) << 1) |
                     ((uint32_t)(nv[r][2] == lo.z) << 2) | ((uint32_t)(nv[r][3] == lo.w) << 3) |
                     ((uint32_t)(nv[r][4] == hi.x) << 4) | ((uint32_t)(nv[r][5] == hi.y) << 5) |
                     ((uint32_t)(nv[r][6] == hi.z) << 6) | ((uint32_t)(nv[r][7] == hi.w) << 7);
        if (paper) {
          // Listing 11: res = lhs if (lhs.id==14 && rhs.id!=14) else rhs
          const bool m14 = m == 0xFFu;
          const bool keep = b14[r] && !m14;
          if (!keep) { bid[r] = id; bmask[r] = m; b14[r] = m14; brank[r] = 0; }
        } else {
          const uint32_t word = srank[(m >> 2) * 32 + lane];
          const int rk = (int)((word >> ((m & 3u) * 8u)) & 0xFFu);
          const bool take = rk > brank[r] || (rk == brank[r] && id > bid[r]);
          if (take) { brank[r] = rk; bid[r] = id; bmask[r] = m; }
        }
      }
    }
  }
#pragma unroll
  for (int r = 0; r < T5_R; ++r) {
    if (!valid[r] || i1 <= i0) continue;
    const uint32_t m = bmask[r];
    const long long id = bid[r];
    const double w = P.wtab[m];
    const int im = m == 0xFFu ? 14 : __popc(m);
    if (P.S == 1) {
      P.oid[P.obase[0] + P.oL[0] * nn[r]] = id;
      P.ow[P.obase[1] + P.oL[1] * nn[r]] = w;
      P.om[P.obase[2] + P.oL[2] * nn[r]] = im;
    } else {
      const int64_t e = (int64_t)s * P.N + nn[r];
      P.pid[e] = id;
      P.pw[e] = w;
      P.pm[e] = im;
    }
  }
}

// fold the S split partials of every n in split order (lhs = lower range), write via ω
__global__ void __launch_bounds__(256) t5_combine(const __grid_constant__ T5Params P) {
  for (int64_t n = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; n < P.N; n += (int64_t)gridDim.x * blockDim.x) {
    PrlRec acc{P.pid[n], P.pw[n], P.pm[n]};
    for (int s = 1; s < P.S; ++s) {
      const int64_t e = (int64_t)s * P.N + n;
      PrlRec r{P.pid[e], P.pw[e], P.pm[e]};
      acc = prl_combine(P.op, acc, r);
    }
    P.oid[P.obase[0] + P.oL[0] * n] = acc.id;
    P.ow[P.obase[1] + P.oL[1] * n] = acc.w;
    P.om[P.obase[2] + P.oL[2] * n] = acc.m;
  }
}

// ------------------------------------------------------------------------ host
mdh_status prepare_t5(Plan* p) {
  // the fast path needs exactly one non-degenerate cc dim (n) and one pw dim (i)
  int nd = -1, id = -1, ncnt = 0, icnt = 0;
  for (int d = 0; d < p->D; ++d) {
    if (p->size[d] == 1) continue;
    if (p->op[d] == MDH_CC) { nd = d; ++ncnt; } else { id = d; ++icnt; }
  }
  bool ok = ncnt <= 1 && icnt <= 1;
  for (int k = 0; k < 8 && ok; ++k) ok &= (id < 0 || p->in[k].acc[0].L[id] == 0) && (nd < 0 || p->in[8 + k].acc[0].L[nd] == 0);
  ok &= (nd < 0 || p->in[16].acc[0].L[nd] == 0);
  if (!ok) {
    p->tmpl = T0_GENERIC;
    p->why = "PRL with a non-standard dimension layout: generic template";
    return prepare_t0(p);
  }
  p->tiles.per_thread = nd;   // remember the dims
  p->tiles.zchunk = id;
  // fp64 weight table W[mask] = Σ_{k=0..7} (bit_k ? wa_k : wd_k), field order (reading C-18)
  double W[256];
  for (int m = 0; m < 256; ++m) {
    double acc = 0.0;
    for (int k = 0; k < 8; ++k) acc = acc + (((m >> k) & 1) ? p->fparams[k] : p->fparams[8 + k]);
    W[m] = acc;
  }
  // dense rank of (mask == 0xFF, W[mask]) — ties get equal ranks (reading C-19)
  std::vector<int> order(256);
  for (int m = 0; m < 256; ++m) order[m] = m;
  auto key_less = [&](int a, int b) {
    bool fa = a == 255, fb = b == 255;
    if (fa != fb) return fb;
    return W[a] < W[b];
  };
  std::sort(order.begin(), order.end(), key_less);
  uint8_t rank[256];
  int r = 0;
  for (int q = 0; q < 256; ++q) {
    if (q > 0 && key_less(order[q - 1], order[q])) ++r;
    rank[order[q]] = (uint8_t)r;
  }
  uint32_t rep[64 * 32];
  for (int w = 0; w < 64; ++w) {
    uint32_t word = (uint32_t)rank[4 * w] | ((uint32_t)rank[4 * w + 1] << 8) | ((uint32_t)rank[4 * w + 2] << 16) |
                    ((uint32_t)rank[4 * w + 3] << 24);
    for (int l = 0; l < 32; ++l) rep[w * 32 + l] = word;
  }
  p->host_const.clear();
  p->tab_off[0] = add_const(p, rep, sizeof(rep));
  p->tab_off[1] = add_const(p, W, sizeof(W));
  // split the DB dim when N alone cannot fill the GPU
  int64_t N = nd >= 0 ? p->size[nd] : 1, I = id >= 0 ? p->size[id] : 1;
  int64_t nblk = (N + T5_THREADS * T5_R - 1) / (T5_THREADS * T5_R);
  int S = 1;
  if (p->tiles.split > 0) S = p->tiles.split;
  else if (nblk < 148 * 4) S = (int)std::min<int64_t>((148 * 4 + nblk - 1) / nblk, 64);
  S = (int)std::max<int64_t>(1, std::min<int64_t>(S, (I + T5_TILE - 1) / T5_TILE));
  if (S > 64) S = 64;
  p->tiles.split = S;
  p->ws_kernel = S > 1 ? (size_t)S * N * (8 + 8 + 4) + 1024 : 0;
  return MDH_OK;
}

mdh_status launch_t5(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st) {
  const char* dc = nullptr;
  MDH_TRY(device_consts(p, &dc));
  const int nd = p.tiles.per_thread, id = p.tiles.zchunk;
  T5Params P;
  memset(&P, 0, sizeof(P));
  for (int k = 0; k < 8; ++k) {
    P.nf[k] = (const uint32_t*)in[k];
    P.df[k] = (const uint32_t*)in[8 + k];
    P.nbase[k] = p.in[k].acc[0].base;
    P.nL[k] = nd >= 0 ? p.in[k].acc[0].L[nd] : 0;
    P.dbase[k] = p.in[8 + k].acc[0].base;
    P.dL[k] = id >= 0 ? p.in[8 + k].acc[0].L[id] : 0;
  }
  P.dbid = (const long long*)in[16];
  P.dbase[8] = p.in[16].acc[0].base;
  P.dL[8] = id >= 0 ? p.in[16].acc[0].L[id] : 0;
  P.N = nd >= 0 ? p.size[nd] : 1;
  P.I = id >= 0 ? p.size[id] : 1;
  P.S = p.tiles.split;
  P.ichunk = (P.I + P.S - 1) / P.S;
  P.op = p.redop == MDH_CC ? MDH_PW_PRL_ARGMAX : p.redop;
  P.rank32 = (const uint8_t*)(dc + p.tab_off[0]);
  P.wtab = (const double*)(dc + p.tab_off[1]);
  P.oid = (long long*)out[0];
  P.ow = (double*)out[1];
  P.om = (int32_t*)out[2];
  for (int b = 0; b < 3; ++b) {
    P.obase[b] = p.out[b].acc[0].base;
    P.oL[b] = nd >= 0 ? p.out[b].acc[0].L[nd] : 0;
  }
  char* w = (char*)ws;
  P.pid = (long long*)w;
  P.pw = (double*)(w + (size_t)P.S * P.N * 8);
  P.pm = (int32_t*)(w + (size_t)P.S * P.N * 16);
  const int64_t nblk = (P.N + T5_THREADS * T5_R - 1) / (T5_THREADS * T5_R);
  t5_kernel<<<(unsigned)(nblk * P.S), T5_THREADS, 0, st>>>(P);
  MDH_TRY(post_launch("t5_kernel"));
  if (P.S > 1) {
    t5_combine<<<(unsigned)std::min<int64_t>((P.N + 255) / 256, 148 * 16), 256, 0, st>>>(P);
    MDH_TRY(post_launch("t5_combine"));
  }
  return MDH_OK;
}

}  // namespace mdh
