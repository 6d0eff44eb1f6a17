// t5_prl.cu — T5: probabilistic record linkage (Listing 11; Fig 3):
// md_hom[N,I](PRL_COMPARE, (cc, pw(prl)))  — every new record n is compared with every
// DB record i and the comparison records are folded with the custom pw operator.
//
// ALU-bound (≈2^34 pair evaluations at the config, ~40 MB of data): each thread keeps
// R new records in registers; the CTA stages DB tiles in shared memory and every thread
// folds its R records over the tile in ascending i (A4, the order-preserving mapping
// required by the non-commutative paper rule, reading C-2).
// f (reading C-18): an 8-bit agreement mask from 8 u32 equality tests; the fold only
// needs the ORDER of (id==14, weight), which the plan precomputes per mask as a dense
// rank (ties equal) in a shared-memory table replicated per lane (conflict-free), so a
// pair costs the 8 equality tests, the table address, one lookup and one compare with
// the running best rank; match_id is read and compared only when a rank reaches the
// best (rare once the best has risen).  The fp64 weight Σ_k (bit_k ? wa_k : wd_k),
// summed in field order, and id_measure are produced only for the final best record.
//
// Packed compares (the fast path).  When every field code of a record is < 2^15 (the
// paper's phonetic codes, dates and postcodes: domains ≤ 8192, reading C-18) the record
// is packed two fields per 32-bit word, code x stored as the fp16 bit pattern
// g(x) = x < 0x7C00 ? x : x + 0x401 — an injection into the non-NaN, non-(−0) fp16
// patterns, where IEEE fp16 equality (no flush-to-zero) is exactly bit equality.  One
// `set.eq.f16x2` (HSET2) then tests two fields, and fp16 arithmetic on its 1.0 / 0.0
// halves builds the rank address (packed_addr): 4 HSET2 + 1 LEA on the ALU pipe and 5
// half-precision FMA/ADDs on the FMA pipe per pair, instead of 8 compares and 8 predicated
// adds all on the ALU pipe (ncu: the ALU pipe, half the issue rate, was the bound).  The
// mask index is permuted — bit j = field 2j, bit 4+j = field 2j+1 (prl_pos) — and the
// rank table is laid out in that order.  A tile (or a CTA's new records) holding a code
// ≥ 2^15 takes the general per-field compares for that tile, with the same permuted
// index, so results never depend on the path.
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
constexpr int T5_R = 4;           // new records per thread (tile knob vec: 4 or 8)
constexpr int T5_R8 = 8;
constexpr int T5_TILE = 512;      // DB records per smem tile

// position of field k's agreement bit in the (permuted) mask index
__host__ __device__ constexpr int prl_pos(int k) { return (k & 1) ? 4 + (k >> 1) : (k >> 1); }

struct T5Params {
  const uint32_t* nf[8];
  const uint32_t* df[8];
  const long long* dbid;
  int64_t nbase[8], nL[8];        // new field k of record n at nbase + nL*n
  int64_t dbase[9], dL[9];        // db field k (k=8: id) of record i at dbase + dL*i
  int64_t N, I, ichunk;
  int S, op;
  const uint32_t* rank32;         // [256][32] words: rank of permuted index x at x*32 + lane
  const double* wtab;             // [256] fp64 weights (natural mask order)
  // outputs: final (through ω) or partials [S][N]
  long long* oid;
  double* ow;
  int32_t* om;
  int64_t obase[3], oL[3];
  long long* pid;
  double* pw;
  int32_t* pm;
};

// fp16 pattern of a field code < 2^15 (see the header); larger codes are not packable
__device__ __forceinline__ uint32_t prl_code16(uint32_t x) { return x < 0x7C00u ? x : x + 0x401u; }

__device__ __forceinline__ uint32_t heq2(uint32_t a, uint32_t b) {     // 1.0 / 0.0 per equal half
  uint32_t m;
  asm("set.eq.f16x2.f16x2 %0, %1, %2;" : "=r"(m) : "r"(a), "r"(b));
  return m;
}
__device__ __forceinline__ uint32_t hfma2(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm("fma.rn.f16x2 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}

// packed compare of new record v and DB record d → shared-memory address of the rank.
// HSET2.BF gives (e_2j, e_2j+1) as fp16 1.0 / 0.0 for word j; three HFMA2s accumulate
// (L, H) = Σ_j 2^j (e_2j, e_2j+1); one HFMA2 folds f = 16·H + L, one HADD2 adds 1024, so
// both halves hold 1024 + x (x = the permuted index, exact in fp16), whose fp16 bit
// pattern is 0x6400 + x; then (f >> 9) = ((0x6400 + x) << 7) + 50 and
// cbase = lanebase − (0x6400 << 7) − 50 gives lanebase + 128·x.  The half ops issue to the
// FMA pipe, the compares to the ALU pipe, so the two halves of the issue rate share the
// work (≈ 5 FMA-pipe + 6 ALU-pipe + 1 LSU instructions per pair).
__device__ __forceinline__ uint32_t packed_addr(const uint4& v, const uint4& d, uint32_t cbase) {
  uint32_t a = hfma2(heq2(v.y, d.y), 0x40004000u, heq2(v.x, d.x));   // + 2·(e2, e3)
  a = hfma2(heq2(v.z, d.z), 0x44004400u, a);                          // + 4·(e4, e5)
  a = hfma2(heq2(v.w, d.w), 0x48004800u, a);                          // + 8·(e6, e7)
  uint32_t hh, ll, f;
  asm("{\n\t.reg .b16 l, h;\n\tmov.b32 {l, h}, %2;\n\tmov.b32 %0, {h, h};\n\tmov.b32 %1, {l, l};\n\t}"
      : "=r"(hh), "=r"(ll) : "r"(a));
  f = hfma2(hh, 0x4C004C00u, ll);                                     // 16·H + L
  asm("add.rn.f16x2 %0, %1, %2;" : "=r"(f) : "r"(f), "r"(0x64006400u));
  return cbase + (f >> 9);
}

// general path: shared-memory address of the rank of the agreement mask of new record v
// and DB record (lo, hi): base + Σ_k [v_k == db_k] · (128 << prl_pos(k)) — a compare and
// a predicated add of the scaled bit per field
__device__ __forceinline__ uint32_t mask_addr(const uint32_t* v, const uint4& lo, const uint4& hi, uint32_t base) {
  uint32_t a = base;
  asm("{\n\t.reg .pred q0, q1, q2, q3, q4, q5, q6, q7;\n\t"
      "setp.eq.u32 q0, %1, %9;\n\tsetp.eq.u32 q1, %2, %10;\n\t"
      "setp.eq.u32 q2, %3, %11;\n\tsetp.eq.u32 q3, %4, %12;\n\t"
      "setp.eq.u32 q4, %5, %13;\n\tsetp.eq.u32 q5, %6, %14;\n\t"
      "setp.eq.u32 q6, %7, %15;\n\tsetp.eq.u32 q7, %8, %16;\n\t"
      "@q0 add.u32 %0, %0, 128;\n\t@q1 add.u32 %0, %0, 2048;\n\t"
      "@q2 add.u32 %0, %0, 256;\n\t@q3 add.u32 %0, %0, 4096;\n\t"
      "@q4 add.u32 %0, %0, 512;\n\t@q5 add.u32 %0, %0, 8192;\n\t"
      "@q6 add.u32 %0, %0, 1024;\n\t@q7 add.u32 %0, %0, 16384;\n\t}"
      : "+r"(a)
      : "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(lo.x), "r"(lo.y),
        "r"(lo.z), "r"(lo.w), "r"(hi.x), "r"(hi.y), "r"(hi.z), "r"(hi.w));
  return a;
}

__device__ __forceinline__ int lds_rank(uint32_t a) {
  int rk;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(rk) : "r"(a));
  return rk;
}

// natural 8-bit mask (bit k = field k) of a permuted index
__device__ __forceinline__ uint32_t prl_unpermute(uint32_t x) {
  uint32_t m = 0;
#pragma unroll
  for (int k = 0; k < 8; ++k) m |= ((x >> prl_pos(k)) & 1u) << k;
  return m;
}

// running best of one new record: rank (ARGMAX) / id14 flag (PAPER), id, permuted index
struct PrlBest {
  int rank;
  long long id;
  uint32_t x;
};

// fold DB record (rank rk, permuted index x, id from sid) into the running best (ARGMAX:
// lexicographic (rank, id); PAPER: Listing 11 — res = lhs if lhs.id==14 && rhs.id!=14
// else rhs, rank field used as the lhs id==14 flag)
__device__ __forceinline__ void paper_step(PrlBest& b, uint32_t x, long long id) {
  const bool m14 = x == 0xFFu;
  if (!(b.rank && !m14)) { b.rank = m14; b.id = id; b.x = x; }
}

// ---- the fold, shared by both kernels: new records bn·R·256 + r·256 + tid, DB range of
// split s = [s·ichunk, min(I, (s+1)·ichunk)), DB tiles staged in shared memory
struct T5Slice {
  int64_t bn, i0, i1;
  int s;
};
template <int R>
__device__ __forceinline__ T5Slice t5_slice(const T5Params& P) {
  const int64_t nblk = (P.N + T5_THREADS * R - 1) / (T5_THREADS * R);
  T5Slice q;
  q.bn = blockIdx.x % nblk;
  q.s = (int)(blockIdx.x / nblk);
  q.i0 = (int64_t)q.s * P.ichunk;
  q.i1 = min(P.I, q.i0 + P.ichunk);
  return q;
}

// write the best record of new record n (final through ω, or the split partial)
__device__ __forceinline__ void t5_emit(const T5Params& P, int s, int64_t n, const PrlBest& b) {
  const uint32_t m = prl_unpermute(b.x);
  const double w = P.wtab[m];
  const int im = m == 0xFFu ? 14 : __popc(m);
  if (P.S == 1) {
    P.oid[P.obase[0] + P.oL[0] * n] = b.id;
    P.ow[P.obase[1] + P.oL[1] * n] = w;
    P.om[P.obase[2] + P.oL[2] * n] = im;
  } else {
    const int64_t e = (int64_t)s * P.N + n;
    P.pid[e] = b.id;
    P.pw[e] = w;
    P.pm[e] = im;
  }
}

// unpackable flag: any field code ≥ 2^15 in the new or DB records (the packed kernel then
// exits at once and the general kernel runs; otherwise the reverse).  *flag is zeroed
// by a memset before this launch.
__global__ void __launch_bounds__(256) t5_check_kernel(const __grid_constant__ T5Params P, unsigned* flag) {
  uint32_t bad = 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t n = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; n < P.N; n += stride)
#pragma unroll
    for (int k = 0; k < 8; ++k) bad |= __ldg(P.nf[k] + P.nbase[k] + P.nL[k] * n);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < P.I; i += stride)
#pragma unroll
    for (int k = 0; k < 8; ++k) bad |= __ldg(P.df[k] + P.dbase[k] + P.dL[k] * i);
  if (__syncthreads_or(bad >= 0x8000u) && threadIdx.x == 0) atomicOr(flag, 1u);
}

// ---- packed kernel (every code < 2^15): fp16 compares, R new records per thread
template <int R, int MINB, int U>
__global__ void __launch_bounds__(T5_THREADS, MINB) t5_kernel(const __grid_constant__ T5Params P,
                                                                 const unsigned* flag) {
  if (*(volatile const unsigned*)flag) return;            // the general kernel runs instead
  __shared__ __align__(16) uint4 spk[T5_TILE];            // packed DB codes
  __shared__ long long sid[T5_TILE];
  extern __shared__ uint32_t srank[];     // [256][32], dynamic (32 KB)
  const int tid = threadIdx.x, lane = tid & 31;
  for (int k = tid; k < 256 * 32; k += T5_THREADS) srank[k] = P.rank32[k];
  const uint32_t lanebase = (uint32_t)__cvta_generic_to_shared(srank) + 4u * lane;
  const uint32_t cbase = lanebase - (0x6400u << 7) - 50u;
  const T5Slice q = t5_slice<R>(P);
  const int64_t n0 = q.bn * (T5_THREADS * R) + tid;
  uint4 nv[R];                            // packed new records
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const int64_t n = n0 + r * T5_THREADS;
    uint32_t f[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) f[k] = prl_code16(n < P.N ? __ldg(P.nf[k] + P.nbase[k] + P.nL[k] * n) : 0u);
    // an absent record holds fp16 NaNs: it never agrees (and is never written)
    nv[r] = n < P.N ? make_uint4(f[0] | f[1] << 16, f[2] | f[3] << 16, f[4] | f[5] << 16, f[6] | f[7] << 16)
                    : make_uint4(~0u, ~0u, ~0u, ~0u);
  }
  const bool paper = P.op == MDH_PW_PRL_PAPER;
  PrlBest b[R];
#pragma unroll
  for (int r = 0; r < R; ++r) b[r] = PrlBest{paper ? 0 : -1, 0, 0};   // PAPER: rank = "lhs.id == 14"
  for (int64_t t0 = q.i0; t0 < q.i1; t0 += T5_TILE) {
    const int cnt = (int)min((int64_t)T5_TILE, (int64_t)(q.i1 - t0));
    __syncthreads();
    for (int j = tid; j < cnt; j += T5_THREADS) {
      const int64_t i = t0 + j;
      uint32_t f[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) f[k] = prl_code16(__ldg(P.df[k] + P.dbase[k] + P.dL[k] * i));
      spk[j] = make_uint4(f[0] | f[1] << 16, f[2] | f[3] << 16, f[4] | f[5] << 16, f[6] | f[7] << 16);
      sid[j] = __ldg(P.dbid + P.dbase[8] + P.dL[8] * i);
    }
    __syncthreads();
    if (!paper) {
#pragma unroll U
      for (int j = 0; j < cnt; ++j) {
        const uint4 d = spk[j];
        uint32_t a[R];
        int rk[R];
        bool any = false;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          a[r] = packed_addr(nv[r], d, cbase);
          rk[r] = lds_rank(a[r]);
        }
#pragma unroll
        for (int r = 0; r < R; ++r) any |= rk[r] >= b[r].rank;
        if (any) {                       // some rank reached the running best: tie-break on id
          const long long id = sid[j];
#pragma unroll
          for (int r = 0; r < R; ++r)
            if (rk[r] > b[r].rank || (rk[r] == b[r].rank && id > b[r].id)) {
              b[r].rank = rk[r];
              b[r].id = id;
              b[r].x = (a[r] - lanebase) >> 7;
            }
        }
      }
    } else {
      for (int j = 0; j < cnt; ++j) {
        const uint4 d = spk[j];
        const long long id = sid[j];
#pragma unroll
        for (int r = 0; r < R; ++r) paper_step(b[r], (packed_addr(nv[r], d, cbase) - lanebase) >> 7, id);
      }
    }
  }
  if (q.i1 <= q.i0) return;
#pragma unroll
  for (int r = 0; r < R; ++r)
    if (n0 + r * T5_THREADS < P.N) t5_emit(P, q.s, n0 + r * T5_THREADS, b[r]);
}

// ---- general kernel (some code ≥ 2^15): per-field u32 compares, same permuted index
template <int R>
__global__ void __launch_bounds__(T5_THREADS, 2) t5_general_kernel(const __grid_constant__ T5Params P,
                                                                   const unsigned* flag) {
  if (!*(volatile const unsigned*)flag) return;           // the packed kernel ran
  __shared__ __align__(16) uint32_t sf[T5_TILE][8];
  __shared__ long long sid[T5_TILE];
  extern __shared__ uint32_t srank[];
  const int tid = threadIdx.x, lane = tid & 31;
  for (int k = tid; k < 256 * 32; k += T5_THREADS) srank[k] = P.rank32[k];
  const uint32_t lanebase = (uint32_t)__cvta_generic_to_shared(srank) + 4u * lane;
  const T5Slice q = t5_slice<R>(P);
  const int64_t n0 = q.bn * (T5_THREADS * R) + tid;
  uint32_t v[R][8];
#pragma unroll
  for (int r = 0; r < R; ++r)
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int64_t n = n0 + r * T5_THREADS;
      v[r][k] = n < P.N ? __ldg(P.nf[k] + P.nbase[k] + P.nL[k] * n) : 0u;
    }
  const bool paper = P.op == MDH_PW_PRL_PAPER;
  PrlBest b[R];
#pragma unroll
  for (int r = 0; r < R; ++r) b[r] = PrlBest{paper ? 0 : -1, 0, 0};
  for (int64_t t0 = q.i0; t0 < q.i1; t0 += T5_TILE) {
    const int cnt = (int)min((int64_t)T5_TILE, (int64_t)(q.i1 - t0));
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
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const uint32_t a = mask_addr(v[r], lo, hi, lanebase);
        const uint32_t x = (a - lanebase) >> 7;
        if (paper) {
          paper_step(b[r], x, sid[j]);
        } else {
          const int rk = lds_rank(a);
          if (rk >= b[r].rank) {
            const long long id = sid[j];
            if (rk > b[r].rank || id > b[r].id) { b[r].rank = rk; b[r].id = id; b[r].x = x; }
          }
        }
      }
    }
  }
  if (q.i1 <= q.i0) return;
#pragma unroll
  for (int r = 0; r < R; ++r)
    if (n0 + r * T5_THREADS < P.N) t5_emit(P, q.s, n0 + r * T5_THREADS, b[r]);
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
// packed kernel variants: R new records per thread (tile knob vec 4 | 8) and the register
// budget sized for MINB resident CTAs per SM (tile knob stages 2 | 3)
static const void* t5_kernel_ptr(int R, bool packed, int minb = 2, int u = 0) {
  if (packed) {
    if (R == T5_R8) return u == 4 ? (const void*)t5_kernel<T5_R8, 2, 4> : u == 8 ? (const void*)t5_kernel<T5_R8, 2, 1>
                                                                        : (const void*)t5_kernel<T5_R8, 2, 2>;
    if (minb == 3) return u == 8 ? (const void*)t5_kernel<T5_R, 3, 8> : (const void*)t5_kernel<T5_R, 3, 4>;
    return u == 2 ? (const void*)t5_kernel<T5_R, 2, 2> : u == 8 ? (const void*)t5_kernel<T5_R, 2, 8>
                                                              : (const void*)t5_kernel<T5_R, 2, 4>;
  }
  return R == T5_R8 ? (const void*)t5_general_kernel<T5_R8> : (const void*)t5_general_kernel<T5_R>;
}

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
  // table row x = the permuted mask index (bit prl_pos(k) = field k), replicated per lane
  std::vector<uint32_t> rep(256 * 32);
  for (int x = 0; x < 256; ++x) {
    int m = 0;
    for (int k = 0; k < 8; ++k) m |= ((x >> prl_pos(k)) & 1) << k;
    for (int l = 0; l < 32; ++l) rep[x * 32 + l] = rank[m];
  }
  p->host_const.clear();
  p->tab_off[0] = add_const(p, rep.data(), rep.size() * sizeof(uint32_t));
  p->tab_off[1] = add_const(p, W, sizeof(W));
  int64_t N = nd >= 0 ? p->size[nd] : 1, I = id >= 0 ? p->size[id] : 1;
  // 4 new records per thread (8: tile knob vec=8 — measured 1147 vs 1466 Gpairs/s on 2^20×2^14)
  // tile knobs (defaults in tiles.cpp): vec = new records per thread (4 | 8), stages = CTAs
  // per SM the registers are budgeted for (2 | 3, R = 4 only), bk = DB-loop unroll (2 | 4 | 8).
  // Measured (prl_A / prl_B, ms): R=4, 3 CTAs/SM, unroll ×4 7.40 / 7.47; 2 CTAs/SM
  // 7.80 / 7.65; unroll ×2 8.04 (3 CTAs) / 8.64 (2 CTAs); ×8 7.90 / 8.37
  const int Rn = p->tiles.vec == 8 ? T5_R8 : T5_R;
  p->tiles.vec = Rn;
  p->tiles.stages = p->tiles.stages == 3 && Rn == T5_R ? 3 : 2;
  p->tiles.bk = (p->tiles.bk == 2 || p->tiles.bk == 8) ? p->tiles.bk : 4;
  int64_t nblk = (N + T5_THREADS * Rn - 1) / (T5_THREADS * Rn);
  // split the DB dim when N alone gives less than two waves of CTAs, choosing S so the
  // CTAs fill whole waves: time ∝ ceil(nblk·S / slots) / S (slots = SMs × resident CTAs),
  // smallest S on ties, I-chunks of at least one tile.  (With ≥ 2 waves the partial last
  // wave costs little — resident CTAs share an SM's issue slots — and splitting measured
  // slower: 2^20×2^14 at S = 13 took 12.96 ms vs 11.72 ms unsplit.)
  int sms = 148, per_sm = 2;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, p->device) != cudaSuccess) { cudaGetLastError(); sms = 148; }
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, t5_kernel_ptr(Rn, true, p->tiles.stages, p->tiles.bk),
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
  // workspace: split partials [S][N] (S > 1), then the 4-byte unpackable flag
  p->ws_kernel = (S > 1 ? ((size_t)S * N * (8 + 8 + 4) + 1023) / 1024 * 1024 : 0) + 256;
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
  unsigned* flag = (unsigned*)(w + p.ws_kernel - 256);
  static std::once_flag once;
  static cudaError_t aerr = cudaSuccess;
  std::call_once(once, [] {
    for (int r : {T5_R, T5_R8})
      for (int v : {0, 2, 3})
        for (int u : {2, 4, 8}) {
          const cudaError_t e = cudaFuncSetAttribute(t5_kernel_ptr(r, v > 0, v, u), cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_RANK);
          if (e != cudaSuccess && aerr == cudaSuccess) aerr = e;
        }
  });
  MDH_CUDA(aerr);
  // every code < 2^15? (one pass over the 16 field arrays; then exactly one of the two fold
  // kernels does the work, the other returns at its first instruction)
  MDH_CUDA(cudaMemsetAsync(flag, 0, sizeof(unsigned), st));
  t5_check_kernel<<<148 * 4, 256, 0, st>>>(P, flag);
  MDH_TRY(post_launch("t5_check_kernel"));
  const unsigned* cflag = flag;
  void* args[2] = {&P, &cflag};
  const dim3 grid((unsigned)(nblk * P.S));
  MDH_CUDA(cudaLaunchKernel(t5_kernel_ptr(Rn, true, p.tiles.stages, p.tiles.bk), grid, dim3(T5_THREADS), args, SMEM_RANK, st));
  MDH_TRY(post_launch("t5_kernel"));
  MDH_CUDA(cudaLaunchKernel(t5_kernel_ptr(Rn, false), grid, dim3(T5_THREADS), args, SMEM_RANK, st));
  MDH_TRY(post_launch("t5_general_kernel"));
  if (P.S > 1) {
    t5_combine<<<(unsigned)std::min<int64_t>((P.N + 255) / 256, 148 * 16), 256, 0, st>>>(P);
    MDH_TRY(post_launch("t5_combine"));
  }
  return MDH_OK;
}

}  // namespace mdh
