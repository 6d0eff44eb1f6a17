// t3_simt.cu — T3: SIMT (CUDA-core FFMA / IMAD) contraction for f = MUL, ⊗ = pw(add)
// with reuse (MatMul fp32, Listing 9; fp32 CCSD(T) Fig 3 P:526-527 and MCC
// Listing 12 P:401-429 parity runs; int32 contractions).
//
// Dimension grouping (A0): M = cc dims only A's index function uses, N = cc dims only
// B uses, Z (batch) = cc dims both use, K = the pw dims.  Because index functions are
// affine, each operand offset separates: offA = offA_Z[z] + offA_M[m] + offA_K[k]
// (likewise B and C); the plan builds these tables once on the host.  This one kernel
// therefore covers MatMul, transposed/batched MatMul, tensor contractions and
// stride-2 convolutions (implicit im2col) alike.
//
// Tiling (A1, A4): 128×128 CTA tile, BK = 8, 256 threads each owning an 8×8 register
// tile; A/B tiles gathered with coalesced loads along whichever of M/K (N/K) is
// contiguous, staged in shared memory (double-buffered through registers).  fp32
// accumulate (reading C-13), int32 wraps (C-12).  Optional split-K over CTAs (A7):
// fp32 partials [S][Z·M·N] folded in split order by the combine kernel.
#include <algorithm>
#include <vector>

#include "kcommon.cuh"

namespace mdh {

enum { T3_TAB_AM = 0, T3_TAB_AK, T3_TAB_BN, T3_TAB_BK, T3_TAB_CM, T3_TAB_CN, T3_TAB_AZ, T3_TAB_BZ, T3_TAB_CZ };

struct T3Params {
  const void* A;
  const void* B;
  void* C;
  int cdt;
  const int64_t* tab[9];
  int64_t M, N, K, Z;
  int64_t kchunk;
  int S;
  int a_kcontig, b_kcontig;
  void* partial;     // V[S][Z][M][N] when S > 1
};

template <class TI, class V>
__device__ __forceinline__ V ldv(const TI* p, int64_t i) {
  if constexpr (std::is_same<TI, uint16_t>::value) return (V)bf16_to_f32(p[i]);
  else return (V)__ldg(p + i);
}

template <class TI, class V>
__global__ void __launch_bounds__(256, 1) t3_kernel(const __grid_constant__ T3Params P) {
  constexpr int BM = 128, BN = 128, BK = 8;
  __shared__ __align__(16) V As[2][BK][BM];
  __shared__ __align__(16) V Bs[2][BK][BN];
  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;
  const int64_t m0 = (int64_t)blockIdx.y * BM, n0 = (int64_t)blockIdx.x * BN;
  const int64_t zs = blockIdx.z;
  const int64_t z = zs % P.Z;
  const int s = (int)(zs / P.Z);
  const int64_t kbeg = (int64_t)s * P.kchunk;
  const int64_t kend = min(P.K, kbeg + P.kchunk);
  const TI* A = (const TI*)P.A + P.tab[T3_TAB_AZ][z];
  const TI* B = (const TI*)P.B + P.tab[T3_TAB_BZ][z];
  const int64_t* aK = P.tab[T3_TAB_AK];
  const int64_t* bK = P.tab[T3_TAB_BK];

  // per-thread load coordinates (fixed rows/cols across k-tiles)
  int la_m[4], la_k[4], lb_n[4], lb_k[4];
  int64_t la_row[4], lb_col[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    if (P.a_kcontig) { la_m[j] = tid >> 1; la_k[j] = (tid & 1) * 4 + j; }
    else { la_k[j] = tid >> 5; la_m[j] = (tid & 31) * 4 + j; }
    if (P.b_kcontig) { lb_n[j] = tid >> 1; lb_k[j] = (tid & 1) * 4 + j; }
    else { lb_k[j] = tid >> 5; lb_n[j] = (tid & 31) * 4 + j; }
    int64_t gm = m0 + la_m[j], gn = n0 + lb_n[j];
    la_row[j] = gm < P.M ? P.tab[T3_TAB_AM][gm] : -1;
    lb_col[j] = gn < P.N ? P.tab[T3_TAB_BN][gn] : -1;
  }
  V ra[4], rb[4];
  auto gload = [&](int64_t k0) {
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int64_t ka = k0 + la_k[j], kb = k0 + lb_k[j];
      ra[j] = (la_row[j] >= 0 && ka < kend) ? ldv<TI, V>(A, la_row[j] + __ldg(aK + ka)) : (V)0;
      rb[j] = (lb_col[j] >= 0 && kb < kend) ? ldv<TI, V>(B, lb_col[j] + __ldg(bK + kb)) : (V)0;
    }
  };
  auto sstore = [&](int buf) {
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      As[buf][la_k[j]][la_m[j]] = ra[j];
      Bs[buf][lb_k[j]][lb_n[j]] = rb[j];
    }
  };
  V acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = (V)0;

  int64_t k0 = kbeg;
  gload(k0);
  sstore(0);
  __syncthreads();
  int buf = 0;
  for (; k0 < kend; k0 += BK) {
    const bool more = k0 + BK < kend;
    if (more) gload(k0 + BK);
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      V a[8], b[8];
      const V* ap = &As[buf][kk][0];
      const V* bp = &Bs[buf][kk][0];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        a[i] = ap[ty * 4 + i];
        a[4 + i] = ap[64 + ty * 4 + i];
        b[i] = bp[tx * 4 + i];
        b[4 + i] = bp[64 + tx * 4 + i];
      }
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = Arith<V>::mul_add(acc[i][j], a[i], b[j]);
    }
    if (more) {
      sstore(buf ^ 1);
      __syncthreads();
      buf ^= 1;
    }
  }
  // epilogue (A8): scatter through the output tables
  const int64_t* cM = P.tab[T3_TAB_CM];
  const int64_t* cN = P.tab[T3_TAB_CN];
  const int64_t cz = P.tab[T3_TAB_CZ][z];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    int64_t gm = m0 + (i < 4 ? ty * 4 + i : 64 + ty * 4 + (i - 4));
    if (gm >= P.M) continue;
    int64_t rowoff = P.S > 1 ? ((z * P.M + gm) * P.N) : (cz + cM[gm]);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      int64_t gn = n0 + (j < 4 ? tx * 4 + j : 64 + tx * 4 + (j - 4));
      if (gn >= P.N) continue;
      if (P.S > 1) ((V*)P.partial)[(int64_t)s * P.Z * P.M * P.N + rowoff + gn] = acc[i][j];
      else store_as<V>(P.C, P.cdt, rowoff + cN[gn], acc[i][j]);
    }
  }
}

// ---- linear fast path (A[m·lda + k], B[k·ldb + n], C[m·ldc + n], fp32, 16-B aligned) ----
// Same 128×128×8 tiling with float4 global loads, float4 shared-memory reads and float4
// stores, no offset tables, ≤128 registers so two CTAs share an SM.
struct T3Lin {
  const float* A;
  const float* B;
  float* C;
  int M, N, K, lda, ldb, ldc;
};

// FP (fragment-pipelined) = true: one CTA per SM (up to 255 registers) and the shared-memory
// fragments of k-step kk+1 loaded into a second register set while the 64 FMAs of k-step kk
// run (no short-scoreboard stall on the LDS results)
// FFMA2 (sm_100 `fma.rn.f32x2`; default, tile knob mode=0: FFMA): the 8×8 accumulators as 32 fp32 pairs
// (32 instead of 64 FMA instructions per k-step, and 126 registers without spills, so two
// CTAs fit an SM),
// acc[i][2j..2j+1] = fma(a_i, b[2j..2j+1], acc) in one instruction — the same per-element
// fp32 FMA sequence (bit-identical results), half the FMA instructions to issue
__device__ __forceinline__ void ffma2(unsigned long long& acc, unsigned long long a2, unsigned long long b2) {
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc) : "l"(a2), "l"(b2));
}
__device__ __forceinline__ unsigned long long pair2(float x, float y) {
  unsigned long long r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(x), "f"(y));
  return r;
}
__device__ __forceinline__ float lo2(unsigned long long v) { return __uint_as_float((unsigned)v); }
__device__ __forceinline__ float hi2(unsigned long long v) { return __uint_as_float((unsigned)(v >> 32)); }

template <bool FP, bool F2 = false>
__global__ void __launch_bounds__(256, FP ? 1 : 2) t3_linear_kernel(const __grid_constant__ T3Lin P) {
  constexpr int KB = FP ? 16 : 8;                 // k-block (FP: half as many barriers)
  constexpr int H = KB / 8;                        // 8-deep slices per k-block
  __shared__ __align__(16) float As[2][KB][128 + 4];
  __shared__ __align__(16) float Bs[2][KB][128];
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int m0 = blockIdx.y * 128, n0 = blockIdx.x * 128;
  const int am = tid >> 1, ak = (tid & 1) * 4;      // A: row am, 4 consecutive k (+8h)
  const int bk = tid >> 5, bn = (tid & 31) * 4;     // B: row bk (+8h), 4 consecutive n
  const bool arow = m0 + am < P.M, bcol = n0 + bn + 3 < P.N;
  const float* Ap = P.A + (int64_t)(m0 + am) * P.lda + ak;
  const float* Bp = P.B + (int64_t)bk * P.ldb + n0 + bn;
  float4 ra[H], rb[H];
  auto gload = [&](int k0) {
#pragma unroll
    for (int h = 0; h < H; ++h) {
      const int kh = k0 + 8 * h;
      ra[h] = make_float4(0.f, 0.f, 0.f, 0.f);
      rb[h] = ra[h];
      if (arow) {
        if (kh + ak + 3 < P.K) ra[h] = __ldg(reinterpret_cast<const float4*>(Ap + kh));
        else {
          float t[4];
          for (int j = 0; j < 4; ++j) t[j] = (kh + ak + j < P.K) ? __ldg(Ap + kh + j) : 0.f;
          ra[h] = make_float4(t[0], t[1], t[2], t[3]);
        }
      }
      if (kh + bk < P.K) {
        const float* b = Bp + (int64_t)kh * P.ldb;
        if (bcol) rb[h] = __ldg(reinterpret_cast<const float4*>(b));
        else {
          float t[4];
          for (int j = 0; j < 4; ++j) t[j] = (n0 + bn + j < P.N) ? __ldg(b + j) : 0.f;
          rb[h] = make_float4(t[0], t[1], t[2], t[3]);
        }
      }
    }
  };
  auto sstore = [&](int buf) {
#pragma unroll
    for (int h = 0; h < H; ++h) {
      As[buf][8 * h + ak + 0][am] = ra[h].x;
      As[buf][8 * h + ak + 1][am] = ra[h].y;
      As[buf][8 * h + ak + 2][am] = ra[h].z;
      As[buf][8 * h + ak + 3][am] = ra[h].w;
      *reinterpret_cast<float4*>(&Bs[buf][8 * h + bk][bn]) = rb[h];
    }
  };
  float acc[8][8];
  unsigned long long acc2[8][4];           // (F2) acc[i][2j], acc[i][2j+1]
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc2[i][j] = 0ull;
  gload(0);
  sstore(0);
  __syncthreads();
  int buf = 0;
  for (int k0 = 0; k0 < P.K; k0 += KB) {
    const bool more = k0 + KB < P.K;
    if (more) gload(k0 + KB);
    if (FP) {
      float4 fa[2][2], fb[2][2];
      fa[0][0] = *reinterpret_cast<const float4*>(&As[buf][0][ty * 4]);
      fa[0][1] = *reinterpret_cast<const float4*>(&As[buf][0][64 + ty * 4]);
      fb[0][0] = *reinterpret_cast<const float4*>(&Bs[buf][0][tx * 4]);
      fb[0][1] = *reinterpret_cast<const float4*>(&Bs[buf][0][64 + tx * 4]);
#pragma unroll
      for (int kk = 0; kk < KB; ++kk) {
        const int cur = kk & 1, nxt = cur ^ 1;
        if (kk < KB - 1) {
          fa[nxt][0] = *reinterpret_cast<const float4*>(&As[buf][kk + 1][ty * 4]);
          fa[nxt][1] = *reinterpret_cast<const float4*>(&As[buf][kk + 1][64 + ty * 4]);
          fb[nxt][0] = *reinterpret_cast<const float4*>(&Bs[buf][kk + 1][tx * 4]);
          fb[nxt][1] = *reinterpret_cast<const float4*>(&Bs[buf][kk + 1][64 + tx * 4]);
        }
        const float a[8] = {fa[cur][0].x, fa[cur][0].y, fa[cur][0].z, fa[cur][0].w,
                            fa[cur][1].x, fa[cur][1].y, fa[cur][1].z, fa[cur][1].w};
        const float b[8] = {fb[cur][0].x, fb[cur][0].y, fb[cur][0].z, fb[cur][0].w,
                            fb[cur][1].x, fb[cur][1].y, fb[cur][1].z, fb[cur][1].w};
        if (F2) {
          unsigned long long b2[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) b2[j] = pair2(b[2 * j], b[2 * j + 1]);
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const unsigned long long a2 = pair2(a[i], a[i]);
#pragma unroll
            for (int j = 0; j < 4; ++j) ffma2(acc2[i][j], a2, b2[j]);
          }
        } else {
#pragma unroll
          for (int i = 0; i < 8; ++i)
#pragma unroll
            for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
        }
      }
    } else {
#pragma unroll
    for (int kk = 0; kk < KB; ++kk) {
      const float4 a0 = *reinterpret_cast<const float4*>(&As[buf][kk][ty * 4]);
      const float4 a1 = *reinterpret_cast<const float4*>(&As[buf][kk][64 + ty * 4]);
      const float4 b0 = *reinterpret_cast<const float4*>(&Bs[buf][kk][tx * 4]);
      const float4 b1 = *reinterpret_cast<const float4*>(&Bs[buf][kk][64 + tx * 4]);
      const float a[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
      const float b[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
      if (F2) {
        unsigned long long b2[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) b2[j] = pair2(b[2 * j], b[2 * j + 1]);
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const unsigned long long a2 = pair2(a[i], a[i]);
#pragma unroll
          for (int j = 0; j < 4; ++j) ffma2(acc2[i][j], a2, b2[j]);
        }
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
      }
    }
    }
    if (more) {
      sstore(buf ^ 1);
      __syncthreads();
      buf ^= 1;
    }
  }
  if (F2) {
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        acc[i][2 * j] = lo2(acc2[i][j]);
        acc[i][2 * j + 1] = hi2(acc2[i][j]);
      }
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int m = m0 + (i < 4 ? ty * 4 + i : 64 + ty * 4 + i - 4);
    if (m >= P.M) continue;
    float* crow = P.C + (int64_t)m * P.ldc;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int n = n0 + h * 64 + tx * 4;
      if (n + 3 < P.N) {
        *reinterpret_cast<float4*>(crow + n) = make_float4(acc[i][4 * h], acc[i][4 * h + 1], acc[i][4 * h + 2], acc[i][4 * h + 3]);
      } else {
        for (int j = 0; j < 4; ++j)
          if (n + j < P.N) crow[n + j] = acc[i][4 * h + j];
      }
    }
  }
}

template <class V>
__global__ void __launch_bounds__(256) t3_splitk_combine(const __grid_constant__ T3Params P) {
  const int64_t total = P.Z * P.M * P.N;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t n = e % P.N, m = (e / P.N) % P.M, z = e / (P.N * P.M);
    V acc = ((const V*)P.partial)[e];
    for (int s = 1; s < P.S; ++s) acc = Arith<V>::add(acc, ((const V*)P.partial)[(int64_t)s * total + e]);   // split order
    store_as<V>(P.C, P.cdt, P.tab[T3_TAB_CZ][z] + P.tab[T3_TAB_CM][m] + P.tab[T3_TAB_CN][n], acc);
  }
}

// ---------------------------------------------------------------------- host
// table of offsets of a dim group, enumerated in row-major (lexicographic) order
static std::vector<int64_t> group_table(const Plan& p, const int* dims, int nd, const Access& acc) {
  int64_t n = 1;
  for (int t = 0; t < nd; ++t) n *= p.size[dims[t]];
  std::vector<int64_t> tab((size_t)n);
  for (int64_t q = 0; q < n; ++q) {
    int64_t rem = q, off = 0;
    for (int t = nd - 1; t >= 0; --t) {
      int64_t v = rem % p.size[dims[t]];
      rem /= p.size[dims[t]];
      off += acc.L[dims[t]] * v;
    }
    tab[(size_t)q] = off;
  }
  return tab;
}

static bool contiguous(const std::vector<int64_t>& t) {
  for (size_t i = 1; i < t.size(); ++i)
    if (t[i] - t[i - 1] != 1) return false;
  return true;
}

// builds the 9 offset tables of a grouped contraction into host_const (shared with T4)
void build_contraction_tables(Plan* p, int64_t* a_kc, int64_t* b_kc) {
  const Contraction& c = p->con;
  const Access& A = p->in[c.a_buf].acc[0];
  const Access& B = p->in[c.b_buf].acc[0];
  const Access& C = p->out[0].acc[0];
  std::vector<int64_t> t[9];
  t[T3_TAB_AM] = group_table(*p, c.md, c.nm, A);
  t[T3_TAB_AK] = group_table(*p, c.kd, c.nk, A);
  t[T3_TAB_BN] = group_table(*p, c.nd, c.nn, B);
  t[T3_TAB_BK] = group_table(*p, c.kd, c.nk, B);
  t[T3_TAB_CM] = group_table(*p, c.md, c.nm, C);
  t[T3_TAB_CN] = group_table(*p, c.nd, c.nn, C);
  t[T3_TAB_AZ] = group_table(*p, c.zd, c.nz, A);
  t[T3_TAB_BZ] = group_table(*p, c.zd, c.nz, B);
  t[T3_TAB_CZ] = group_table(*p, c.zd, c.nz, C);
  for (int k = 0; k < 9; ++k) {
    t[k][0] += 0;
    if (k == T3_TAB_AZ) for (auto& v : t[k]) v += A.base;
    if (k == T3_TAB_BZ) for (auto& v : t[k]) v += B.base;
    if (k == T3_TAB_CZ) for (auto& v : t[k]) v += C.base;
    p->tab_off[k] = add_const(p, t[k].data(), t[k].size() * sizeof(int64_t));
  }
  *a_kc = contiguous(t[T3_TAB_AK]);
  *b_kc = contiguous(t[T3_TAB_BK]);
}

mdh_status prepare_t3(Plan* p) {
  const Contraction& c = p->con;
  bool same = p->in[0].dtype == p->in[1].dtype;
  if (!same || (c.nm + c.nn + c.nk + c.nz) == 0 || p->n_out != 1) {
    p->tmpl = T0_GENERIC;
    p->why = "contraction outside the T3 catalog: generic template";
    return prepare_t0(p);
  }
  int64_t akc, bkc;
  p->host_const.clear();
  build_contraction_tables(p, &akc, &bkc);
  p->tiles.vec = (int)(akc | (bkc << 1));
  // split-K when the output tile grid cannot fill the GPU
  int64_t tiles = ((c.M + 127) / 128) * ((c.N + 127) / 128) * c.Z;
  int S = 1;
  if (p->tiles.split > 0) S = p->tiles.split;
  else if (tiles < 148 && c.K >= 256) S = (int)std::min<int64_t>(std::max<int64_t>(1, 296 / tiles), c.K / 64);
  if (S < 1) S = 1;
  int64_t kchunk = (c.K + S - 1) / S;
  kchunk = (kchunk + 7) / 8 * 8;
  S = (int)((c.K + kchunk - 1) / kchunk);
  p->tiles.split = S;
  p->tiles.bk = (int)std::min<int64_t>(kchunk, INT32_MAX);
  p->ws_kernel = S > 1 ? (size_t)S * c.Z * c.M * c.N * sizeof(float) : 0;
  // linear fast path: fp32 A[m·lda + k], B[k·ldb + n], C[m·ldc + n], all 16-byte aligned
  p->auxi.clear();
  if (S == 1 && c.Z == 1 && p->in[c.a_buf].dtype == MDH_F32 && p->in[c.b_buf].dtype == MDH_F32 &&
      p->out[0].dtype == MDH_F32 && c.M < INT32_MAX && c.N < INT32_MAX && c.K < INT32_MAX) {
    const Access& A = p->in[c.a_buf].acc[0];
    const Access& B = p->in[c.b_buf].acc[0];
    const Access& C = p->out[0].acc[0];
    auto lin = [&](const int* dims, int nd, const Access& acc, int64_t* s) {
      std::vector<int64_t> t = group_table(*p, dims, nd, acc);
      *s = t.size() > 1 ? t[1] - t[0] : 1;
      for (size_t i = 1; i < t.size(); ++i)
        if (t[i] - t[i - 1] != *s) return false;
      return true;
    };
    int64_t sam, sak, sbk, sbn, scm, scn;
    bool ok = lin(c.md, c.nm, A, &sam) && lin(c.kd, c.nk, A, &sak) && lin(c.kd, c.nk, B, &sbk) &&
              lin(c.nd, c.nn, B, &sbn) && lin(c.md, c.nm, C, &scm) && lin(c.nd, c.nn, C, &scn);
    if (c.K == 1) sak = 1;
    if (c.N == 1) sbn = scn = 1;
    if (c.M == 1) sam = scm = 4;
    if (c.K == 1) sbk = 4;
    ok = ok && sak == 1 && sbn == 1 && scn == 1 && sam % 4 == 0 && sbk % 4 == 0 && scm % 4 == 0 && A.base % 4 == 0 &&
         B.base % 4 == 0 && C.base % 4 == 0 && sam < INT32_MAX && sbk < INT32_MAX && scm < INT32_MAX;
    if (ok) p->auxi = {1, sam, sbk, scm, A.base, B.base, C.base};
  }
  return MDH_OK;
}

mdh_status launch_t3(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st) {
  if (!p.auxi.empty() && p.auxi[0] == 1) {
    const Contraction& c = p.con;
    T3Lin L;
    L.A = (const float*)in[c.a_buf] + p.auxi[4];
    L.B = (const float*)in[c.b_buf] + p.auxi[5];
    L.C = (float*)out[0] + p.auxi[6];
    L.M = (int)c.M;
    L.N = (int)c.N;
    L.K = (int)c.K;
    L.lda = (int)p.auxi[1];
    L.ldb = (int)p.auxi[2];
    L.ldc = (int)p.auxi[3];
    dim3 grid((unsigned)((c.N + 127) / 128), (unsigned)((c.M + 127) / 128));
    if (grid.y > 65535) { set_error("T3: grid too large"); return MDH_ERR_UNSUPPORTED; }
    // default: two 128-register CTAs per SM, 8-deep k-blocks, accumulators as FFMA2 pairs
    // (MatMul 4096³ fp32 2.694 ms = 0.71 of the measured FFMA peak; with FFMA 3.795 ms — it
    // spilled); tile knob stages=2: one CTA per SM with 16-deep k-blocks and the next
    // k-step's fragments prefetched into a second register set (2.897 / FFMA 2.936 ms);
    // tile knob mode=0: the FFMA form of either
    const bool f2 = p.tiles.mode != 0;
    if (p.tiles.stages == 2) {
      if (f2) t3_linear_kernel<true, true><<<grid, 256, 0, st>>>(L);
      else t3_linear_kernel<true><<<grid, 256, 0, st>>>(L);
    } else {
      if (f2) t3_linear_kernel<false, true><<<grid, 256, 0, st>>>(L);
      else t3_linear_kernel<false><<<grid, 256, 0, st>>>(L);
    }
    return post_launch("t3_linear_kernel");
  }
  const char* dc = nullptr;
  MDH_TRY(device_consts(p, &dc));
  const Contraction& c = p.con;
  T3Params P;
  memset(&P, 0, sizeof(P));
  P.A = in[c.a_buf];
  P.B = in[c.b_buf];
  P.C = out[0];
  P.cdt = p.out[0].dtype;
  for (int k = 0; k < 9; ++k) P.tab[k] = (const int64_t*)(dc + p.tab_off[k]);
  P.M = c.M;
  P.N = c.N;
  P.K = c.K;
  P.Z = c.Z;
  P.S = p.tiles.split;
  P.kchunk = p.tiles.bk;
  P.a_kcontig = p.tiles.vec & 1;
  P.b_kcontig = (p.tiles.vec >> 1) & 1;
  P.partial = ws;
  dim3 grid((unsigned)((c.N + 127) / 128), (unsigned)((c.M + 127) / 128), (unsigned)(c.Z * P.S));
  if (grid.y > 65535 || grid.z > 65535) { set_error("T3 grid too large"); return MDH_ERR_UNSUPPORTED; }
  mdh_dtype t = p.in[c.a_buf].dtype;
  if (t == MDH_F32) t3_kernel<float, float><<<grid, 256, 0, st>>>(P);
  else if (t == MDH_BF16) t3_kernel<uint16_t, float><<<grid, 256, 0, st>>>(P);
  else if (t == MDH_I32) t3_kernel<int32_t, int32_t><<<grid, 256, 0, st>>>(P);
  else if (t == MDH_U32) t3_kernel<uint32_t, uint32_t><<<grid, 256, 0, st>>>(P);
  else { set_error("T3: unsupported dtype"); return MDH_ERR_UNSUPPORTED; }
  MDH_TRY(post_launch("t3_kernel"));
  if (P.S > 1) {
    int64_t total = c.Z * c.M * c.N;
    unsigned g = (unsigned)std::min<int64_t>((total + 255) / 256, 148LL * 32);
    if (p.compute == MDH_F32) t3_splitk_combine<float><<<g, 256, 0, st>>>(P);
    else if (p.compute == MDH_I32) t3_splitk_combine<int32_t><<<g, 256, 0, st>>>(P);
    else t3_splitk_combine<uint32_t><<<g, 256, 0, st>>>(P);
    MDH_TRY(post_launch("t3_splitk_combine"));
  }
  return MDH_OK;
}

}  // namespace mdh
