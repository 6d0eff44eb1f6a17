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
// rank (ties equal), so a pair costs the 8 compares — each selecting its bit already
// scaled to the table stride and summed onto the lane's table base, so the sum IS the
// shared-memory address — one conflict-free lookup (the rank table is replicated per
// lane/bank) and one compare with the running best rank; match_id is read and compared
// only when the ranks tie (rare once the best has risen).  The fp64 weight Σ_k (bit_k ? wa_k : wd_k), summed in
// field order, and id_measure are produced only for the final best record.
// The reduction dim is split over CTAs when N alone cannot fill the GPU (orientation
// B, 2^14 × 2^20; reading C-20): partial records [S][N] are folded in split order by
// a combine kernel (A7), lhs = lower range.
#include <algorithm>
#include <vector>
#include <mutex>

#include "kcommon.cuh"
#include "prl_common.cuh"

namespace mdh {

constexpr int T5_THREADS = 256;
constexpr int T5_R = 4;           // new records per thread (T5_R8 = 8 when N fills the GPU)
constexpr int T5_R8 = 8;
constexpr int T5_TILE = 512;      // DB records per smem tile

struct T5Params {
  const uint32_t* nf[8];
  const uint32_t* df[8];
  const long long* dbid;
  int64_t nbase[8], nL[8];        // new field k of record n at nbase + nL*n
  int64_t dbase[9], dL[9];        // db field k (k=8: id) of record i at dbase + dL*i
  int64_t N, I, ichunk;
  int S, op;
  const uint32_t* rank32;         // [256][32] words: rank of mask m at m*32 + lane
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

// shared-memory address of the rank of the agreement mask of new record v and DB record
// (lo, hi): base + Σ_k [v_k == db_k] · (128 << k) — compare + select per field, the
// selects summed three at a time
__device__ __forceinline__ uint32_t mask_addr(const uint32_t* v, const uint4& lo, const uint4& hi, uint32_t base) {
  // compare, then a predicated add of the scaled bit onto the running address: 2 ops/field
  uint32_t a = base;
  asm("{\n\t.reg .pred q0, q1, q2, q3, q4, q5, q6, q7;\n\t"
      "setp.eq.u32 q0, %1, %9;\n\tsetp.eq.u32 q1, %2, %10;\n\t"
      "setp.eq.u32 q2, %3, %11;\n\tsetp.eq.u32 q3, %4, %12;\n\t"
      "setp.eq.u32 q4, %5, %13;\n\tsetp.eq.u32 q5, %6, %14;\n\t"
      "setp.eq.u32 q6, %7, %15;\n\tsetp.eq.u32 q7, %8, %16;\n\t"
      "@q0 add.u32 %0, %0, 128;\n\t@q1 add.u32 %0, %0, 256;\n\t"
      "@q2 add.u32 %0, %0, 512;\n\t@q3 add.u32 %0, %0, 1024;\n\t"
      "@q4 add.u32 %0, %0, 2048;\n\t@q5 add.u32 %0, %0, 4096;\n\t"
      "@q6 add.u32 %0, %0, 8192;\n\t@q7 add.u32 %0, %0, 16384;\n\t}"
      : "+r"(a)
      : "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(lo.x), "r"(lo.y),
        "r"(lo.z), "r"(lo.w), "r"(hi.x), "r"(hi.y), "r"(hi.z), "r"(hi.w));
  return a;
}

template <int R>
__global__ void __launch_bounds__(T5_THREADS) t5_kernel(const __grid_constant__ T5Params P) {
  constexpr int T5_R = R;
  __shared__ __align__(16) uint32_t sf[T5_TILE][8];
  __shared__ long long sid[T5_TILE];
  extern __shared__ uint32_t srank[];     // [256][32], dynamic (32 KB)
  const int tid = threadIdx.x, lane = tid & 31;
  for (int k = tid; k < 256 * 32; k += T5_THREADS) srank[k] = P.rank32[k];
  const uint32_t lanebase = (uint32_t)__cvta_generic_to_shared(srank) + 4u * lane;
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
      if (paper) {
        const long long id = sid[j];
#pragma unroll
        for (int r = 0; r < T5_R; ++r) {
          uint32_t m = (uint32_t)(nv[r][0] == lo.x) | ((uint32_t)(nv[r][1] == lo.y) << 1) |
                       ((uint32_t)(nv[r][2] == lo.z) << 2) | ((uint32_t)(nv[r][3] == lo.w) << 3) |
                       ((uint32_t)(nv[r][4] == hi.x) << 4) | ((uint32_t)(nv[r][5] == hi.y) << 5) |
                       ((uint32_t)(nv[r][6] == hi.z) << 6) | ((uint32_t)(nv[r][7] == hi.w) << 7);
          // Listing 11: res = lhs if (lhs.id==14 && rhs.id!=14) else rhs
          const bool m14 = m == 0xFFu;
          const bool keep = b14[r] && !m14;
          if (!keep) { bid[r] = id; bmask[r] = m; b14[r] = m14; brank[r] = 0; }
        }
      } else {
        uint32_t a[T5_R];
        int rk[T5_R];
        bool any = false;
#pragma unroll
        for (int r = 0; r < T5_R; ++r) {
          a[r] = mask_addr(nv[r], lo, hi, lanebase);
          asm("ld.shared.u32 %0, [%1];" : "=r"(rk[r]) : "r"(a[r]));
        }
#pragma unroll
        for (int r = 0; r < T5_R; ++r) any |= rk[r] >= brank[r];
        if (any) {                       // some rank reached the running best: tie-break on id
          const long long id = sid[j];
#pragma unroll
          for (int r = 0; r < T5_R; ++r)
            if (rk[r] > brank[r] || (rk[r] == brank[r] && id > bid[r])) {
              brank[r] = rk[r];
              bid[r] = id;
              bmask[r] = (a[r] - lanebase) >> 7;
            }
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
  std::vector<uint32_t> rep(256 * 32);
  for (int m = 0; m < 256; ++m)
    for (int l = 0; l < 32; ++l) rep[m * 32 + l] = rank[m];
  p->host_const.clear();
  p->tab_off[0] = add_const(p, rep.data(), rep.size() * sizeof(uint32_t));
  p->tab_off[1] = add_const(p, W, sizeof(W));
  int64_t N = nd >= 0 ? p->size[nd] : 1, I = id >= 0 ? p->size[id] : 1;
  // 4 new records per thread (8: tile knob vec=8 — measured 1147 vs 1466 Gpairs/s on 2^20×2^14)
  int Rn = T5_R;
  if (p->tiles.source.find("forced") != std::string::npos && p->tiles.vec == 8) Rn = T5_R8;
  p->tiles.vec = Rn;
  int64_t nblk = (N + T5_THREADS * Rn - 1) / (T5_THREADS * Rn);
  // split the DB dim when N alone gives less than two waves of CTAs, choosing S so the
  // CTAs fill whole waves: time ∝ ceil(nblk·S / slots) / S (slots = SMs × resident CTAs),
  // smallest S on ties, I-chunks of at least one tile.  (With ≥ 2 waves the partial last
  // wave costs little — resident CTAs share an SM's issue slots — and splitting measured
  // slower: 2^20×2^14 at S = 13 took 12.96 ms vs 11.72 ms unsplit.)
  int sms = 148, per_sm = 2;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, p->device) != cudaSuccess) { cudaGetLastError(); sms = 148; }
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, Rn == T5_R8 ? (const void*)t5_kernel<T5_R8> : (const void*)t5_kernel<T5_R>,
                                                    T5_THREADS, 256 * 32 * 4) != cudaSuccess || per_sm < 1) {
    cudaGetLastError();
    per_sm = 2;
  }
  const int64_t slots = (int64_t)sms * per_sm;
  const int smax = (int)std::max<int64_t>(1, std::min<int64_t>(64, (I + T5_TILE - 1) / T5_TILE));
  int S = 1;
  if (p->tiles.split > 0) {
    S = std::min(p->tiles.split, smax);
  } else if (nblk < 2 * slots) {
    double best = 1e30;
    for (int c = 1; c <= smax; ++c) {
      const double t = (double)((nblk * c + slots - 1) / slots) / c;
      if (t < best * (1 - 1e-9)) { best = t; S = c; }
    }
  }
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
  P.rank32 = (const uint32_t*)(dc + p.tab_off[0]);
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
  const int Rn = p.tiles.vec == T5_R8 ? T5_R8 : T5_R;
  const int64_t nblk = (P.N + T5_THREADS * Rn - 1) / (T5_THREADS * Rn);
  constexpr int SMEM_RANK = 256 * 32 * 4;
  static std::once_flag once;
  static cudaError_t aerr = cudaSuccess;
  std::call_once(once, [] {
    cudaError_t e1 = cudaFuncSetAttribute((const void*)t5_kernel<T5_R>, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_RANK);
    cudaError_t e2 = cudaFuncSetAttribute((const void*)t5_kernel<T5_R8>, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_RANK);
    aerr = e1 != cudaSuccess ? e1 : e2;
  });
  MDH_CUDA(aerr);
  if (Rn == T5_R8) t5_kernel<T5_R8><<<(unsigned)(nblk * P.S), T5_THREADS, SMEM_RANK, st>>>(P);
  else t5_kernel<T5_R><<<(unsigned)(nblk * P.S), T5_THREADS, SMEM_RANK, st>>>(P);
  MDH_TRY(post_launch("t5_kernel"));
  if (P.S > 1) {
    t5_combine<<<(unsigned)std::min<int64_t>((P.N + 255) / 256, 148 * 16), 256, 0, st>>>(P);
    MDH_TRY(post_launch("t5_combine"));
  }
  return MDH_OK;
}

}  // namespace mdh
