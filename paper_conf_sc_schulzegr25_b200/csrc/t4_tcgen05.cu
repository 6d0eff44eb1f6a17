// t4_tcgen05.cu — T4: bf16 contraction on the 5th-generation tensor cores (tcgen05/TMEM)
// for f = MUL, ⊗ = pw(add) with reuse (MatMul Listing 9).
//
// Persistent, warp-specialised sm_100a kernel, one CTA per SM:
//   warp 0       — TMA producer: cp.async.bulk.tensor 2-D loads of the A (128×64) and
//                  B (64×256) bf16 tiles into a 4-stage 128-byte-swizzled smem ring,
//                  completion counted on per-stage mbarriers (expect_tx);
//   warp 1       — TMEM allocator + MMA issuer: one thread issues
//                  tcgen05.mma.cta_group::1.kind::f16 (128×256×16, fp32 accumulate in
//                  TMEM) on UMMA smem descriptors; tcgen05.commit frees smem stages and
//                  signals the epilogue;
//   warps 2..5   — epilogue: tcgen05.ld 32x32b.x32 TMEM → registers → global (fp32),
//                  TMEM double-buffered (2 × 256 columns) so the epilogue of tile t
//                  overlaps the MMAs of tile t+1.
// Operands are described by 2-D tensor maps: an operand qualifies when its M (N) and K
// offset tables are linear with one unit stride (K-major or MN-major; both are native
// UMMA layouts for bf16).  M/N/K tails are TMA out-of-bounds zero fill + masked stores.
// The output goes through the plan's offset tables (any affine out_view, e.g. the
// 6-D CCSD(T) scatter) or, for a row-major C, as 16-byte vector stores.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "kcommon.cuh"

namespace mdh {

void build_contraction_tables(Plan* p, int64_t* a_kc, int64_t* b_kc);

namespace t4 {

constexpr int BM = 128, BN = 256, BK = 64, STAGES = 4;
constexpr int THREADS = 320;                 // 2 control warps + 8 epilogue warps
constexpr int A_BYTES = BM * BK * 2;          // 16 KB
constexpr int B_BYTES = BN * BK * 2;          // 32 KB
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 + 256;
constexpr uint32_t TMEM_COLS = 512;           // 2 accumulators × 256 fp32 columns

// Implicit-GEMM ("box") operand: the tile's rows run along one group dim g* (unit
// coefficient, tile never crosses a g* run), the k-block along one K dim k* (unit
// coefficient on the innermost buffer coordinate); every other dim of the group / of K
// only moves the box origin.  coord[j] = base[j] + Σ_o gco[o][j]·idx_o + Σ_q kco[q][j]·idx_q
// (+ g0 on coordinate jg, + k0 on jk); coordinates in TMA order (innermost first).
struct BoxGen {
  int rank, jg, jk, ng, nk;
  int64_t gsize, ksize;              // extents of g* and k*
  int64_t gdim[4], kdim[4];          // extents of the other group / K dims (outer first)
  int gco[4][5], kco[4][5];
  int base[5];
};

struct Params {
  int a_box;
  BoxGen abox;
  int64_t M, N, K;
  int tiles_m, tiles_n, num_tiles, num_kb;
  int a_mn_major, b_mn_major;
  uint32_t idesc;
  float* C;
  int out_bf16;
  int c_rowmajor;                   // C[m*ldc + n] fast path
  int64_t ldc, cbase;
  const int64_t* cM;                // generic output tables
  const int64_t* cN;
  int sched;                        // 0: round-robin, M-major; 1: contiguous range per CTA, N-major
  // 2-SM split-K tail: units [0, nfull) are whole tiles; the remaining tiles are split into
  // ssplit contiguous k-ranges each (units nfull + i·ssplit + s) whose fp32 partial tiles go
  // to `part` and are folded in split order by tail_combine_kernel
  int nunits, nfull, ssplit;
  float* part;
  unsigned* tail_cnt;               // 2 counters per split tile (arrivals, departures); zero at rest
  // gather producer for A (AG kernels): A[m, k] = Ag[aM[m] + akoff[k/8] + k%8], K % 8 == 0
  const uint16_t* Ag;
  const int64_t* aM;
  const int64_t* aK;                // offA_K table (every 8th entry is a chunk start)
  int nkc;                          // K / 8 (K / 4 with ag4) chunk offsets staged in shared memory
  int ag4;                          // gather in 8-byte runs of 4 (K offsets contiguous in runs of 4)
  int run4;                         // EPI 2 with runs of 4 (fp32: 16-byte stores) instead of 8
  int ag_lag;                       // k-blocks between issuing a stage and publishing it (1..3)
  // bulk-run epilogue (EPI 3): N-tile = 2 output runs of bn/2 contiguous elements
  int bn;                           // N-tile width (EPI 3; else BN)
  int nstg;                         // staging buffers per epilogue warp (1 or 2)
  int e3flip;                       // EPI 3 bank-conflict-free staging order (tile knob epi=2: off)
  int bres;                         // EPI 3: B of the current N-tile resident in shared memory
  // A via TMA im2col (convolution operands, MCC Listing 12): A[(n,p,q), (r,s,c)] =
  // img[n, σh·p + r, σw·q + s, c]; the tensor map walks 128 output pixels (q, then p, then
  // n) with traversal strides (σw, σh) and applies the filter tap (s, r) as im2col offsets
  int a_im2col;
  int ic_C, ic_P, ic_Q, ic_S, ic_sh, ic_sw;
  // k-block rotation: tile t walks its k-range starting at a t-dependent offset, so the
  // CTAs of a wave do not all request the same B rows (MCC: 49 M-tiles share each filter
  // tile) from the same L2 lines at the same time; the fp32 sum order changes only
  int krot;
  // 2-SM stream-K hybrid: tiles [0, nfull) data-parallel (round-robin over the pairs), then
  // the (tile, k-block) space of the remaining tiles, sk_w = (num_tiles - nfull)·num_kb
  // k-blocks, cut into sk_pairs equal contiguous ranges, one per pair (0 = off)
  int sk_pairs;
  int64_t sk_w;
  // column-unit stream (wide 2-SM kernel, vmode): the output is cut into 256-row strips and
  // 128-column units (ups per strip, vunits in all); pair p owns units
  // [p·vunits/npairs, (p+1)·vunits/npairs) — whole K, no partial sums — as tiles of ≤ 4
  // units that never cross a strip, so the pairs' work differs by at most one unit
  int areuse;                       // wide tiles: k-outer MMA order with A kept in the collector
  int vmode, ups;
  int64_t vunits;
  uint32_t idesc128;                // the N = 128 instruction descriptor (a tile's odd last unit)
  float* skpart;                    // one fp32 256×256 partial tile per pair (coalesced layout)
  unsigned* skflag;                 // 16 flags per pair (2 CTAs × 8 epilogue warps); zero at rest
  // diagnostics: per-unit timeline (MDH_T4_TRACE=1; 2-SM kernel), 4 u64 per unit:
  // {smid << 32 | cluster, first MMA issue, last commit, epilogue done} in ns (%globaltimer)
  unsigned long long* trace;
  int trace_n;                      // units the trace buffer holds
  int c_vec4;                       // row-major C with ldc, cbase ≡ 0 mod 4 and a 16-byte base
  int xfold;                        // 1-SM split-K over few tiles: every split writes its partial,
                                    // t4_xfold_kernel folds them in split order afterwards
};

constexpr int AG_WARPS = 4, AG_THREADS = AG_WARPS * 32, KOFF_MAX = 2048;
constexpr int SMEM_AG_BYTES = STAGES * STAGE_BYTES + 1024 + 256 + KOFF_MAX * 8;
constexpr size_t SMEM_LIMIT = 232448;          // 227 KB per CTA (static + dynamic)
constexpr int EPI3_LMAX = 128;                 // longest output run the bulk-run epilogue takes


__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned smid() {
  unsigned r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

__device__ __forceinline__ int krotate(const Params& P, int kb, int kb0, int kb1, int salt) {
  if (!P.krot) return kb;
  const int n = kb1 - kb0;
  return kb0 + (kb - kb0 + (salt * 5) % n) % n;
}

__device__ __forceinline__ void unit_decode(const Params& P, int u, int* t, int* kb0, int* kb1, int* slot) {
  if (u < P.nfull) {
    *t = u; *kb0 = 0; *kb1 = P.num_kb; *slot = -1;
  } else {
    const int v = u - P.nfull, i = v / P.ssplit, s = v % P.ssplit;
    *t = P.nfull + i;
    *kb0 = (int)((int64_t)s * P.num_kb / P.ssplit);
    *kb1 = (int)((int64_t)(s + 1) * P.num_kb / P.ssplit);
    *slot = v;
  }
}

// Tile schedule shared by the three roles.  Round-robin M-major keeps concurrently running
// CTAs on neighbouring tiles (operand reuse in L2); the contiguous N-major range keeps one
// CTA on the same N-tile for many consecutive tiles, so the scatter epilogue caches that
// tile's column offsets in shared memory.
__device__ __forceinline__ int t_first(const Params& P) {
  return P.sched ? (int)((int64_t)blockIdx.x * P.num_tiles / gridDim.x) : (int)blockIdx.x;
}
__device__ __forceinline__ int t_last(const Params& P) {
  return P.sched ? (int)((int64_t)(blockIdx.x + 1) * P.num_tiles / gridDim.x) : P.num_tiles;
}
__device__ __forceinline__ int t_step(const Params& P) { return P.sched ? 1 : (int)gridDim.x; }
__device__ __forceinline__ void t_decode(const Params& P, int t, int* mb, int* nb) {
  if (P.sched) { *nb = t / P.tiles_m; *mb = t % P.tiles_m; }
  else { *mb = t / P.tiles_n; *nb = t % P.tiles_n; }
}
// 1-SM work units: whole tiles (ssplit ≤ 1, schedule above), or with a split-K tail the
// units of unit_decode, round-robin (host sets sched = 0)
__device__ __forceinline__ int u_first(const Params& P) { return P.ssplit > 1 ? (int)blockIdx.x : t_first(P); }
__device__ __forceinline__ int u_last(const Params& P) { return P.ssplit > 1 ? P.nunits : t_last(P); }
__device__ __forceinline__ int u_step(const Params& P) { return P.ssplit > 1 ? (int)gridDim.x : t_step(P); }
__device__ __forceinline__ void u_decode(const Params& P, int u, int* mb, int* nb, int* kb0, int* kb1, int* slot) {
  int t = u;
  if (P.ssplit > 1) unit_decode(P, u, &t, kb0, kb1, slot);
  else { *kb0 = 0; *kb1 = P.num_kb; *slot = -1; }
  t_decode(P, t, mb, nb);
}
__device__ __forceinline__ void named_sync(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1)
      : "memory");
}
// im2col A tile: coordinates of the first output pixel's window origin and the tap offsets
__device__ __forceinline__ void im2col_coords(const Params& P, int64_t m0, int k0, int* c, uint16_t* off) {
  const int64_t pq = (int64_t)P.ic_P * P.ic_Q;
  const int n = (int)(m0 / pq), rem = (int)(m0 % pq);
  const int p = rem / P.ic_Q, q = rem % P.ic_Q;
  const int sc = P.ic_S * P.ic_C;
  const int r = k0 / sc, s = (k0 / P.ic_C) % P.ic_S;
  c[0] = k0 % P.ic_C;
  c[1] = P.ic_sw * q;
  c[2] = P.ic_sh * p;
  c[3] = n;
  off[0] = (uint16_t)s;
  off[1] = (uint16_t)r;
}
__device__ __forceinline__ void tma_load_im2col(uint32_t dst, const CUtensorMap* map, uint32_t bar, const int* c,
                                                const uint16_t* off) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};" ::"r"(dst),
      "l"((uint64_t)map), "r"(bar), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]), "h"(off[0]), "h"(off[1])
      : "memory");
}
__device__ __forceinline__ void tma_load_nd(uint32_t dst, const CUtensorMap* map, uint32_t bar, int rank, const int* c) {
  const uint64_t m = (uint64_t)map;
  switch (rank) {
    case 3:
      asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];"
                   ::"r"(dst), "l"(m), "r"(bar), "r"(c[0]), "r"(c[1]), "r"(c[2]) : "memory");
      break;
    case 4:
      asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];"
                   ::"r"(dst), "l"(m), "r"(bar), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]) : "memory");
      break;
    case 5:
      asm volatile("cp.async.bulk.tensor.5d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6, %7}], [%2];"
                   ::"r"(dst), "l"(m), "r"(bar), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]), "r"(c[4]) : "memory");
      break;
    default:
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                   ::"r"(dst), "l"(m), "r"(bar), "r"(c[0]), "r"(c[1]) : "memory");
  }
}

// box origin of the A tile starting at row m0 (group-linear index) and K offset k0
__device__ __forceinline__ void box_coords(const BoxGen& B, int64_t m0, int64_t k0, int* c) {
#pragma unroll
  for (int j = 0; j < 5; ++j) c[j] = B.base[j];
  int64_t go = m0 / B.gsize;
  c[B.jg] += (int)(m0 % B.gsize);
  for (int o = B.ng - 1; o >= 0; --o) {
    const int v = (int)(go % B.gdim[o]);
    go /= B.gdim[o];
#pragma unroll
    for (int j = 0; j < 5; ++j) c[j] += B.gco[o][j] * v;
  }
  int64_t ko = k0 / B.ksize;
  c[B.jk] += (int)(k0 % B.ksize);
  for (int q = B.nk - 1; q >= 0; --q) {
    const int v = (int)(ko % B.kdim[q]);
    ko /= B.kdim[q];
#pragma unroll
    for (int j = 0; j < 5; ++j) c[j] += B.kco[q][j] * v;
  }
}

// UMMA shared-memory descriptor (sm_100): start>>4 [0,14), LBO>>4 [16,30), SBO>>4 [32,46),
// version 1 [46,48), base offset 0, layout SWIZZLE_128B = 2 at [61,64).
__device__ __forceinline__ uint64_t sdesc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46) | (2ull << 61);
}
__device__ __forceinline__ void mma_bf16(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void mma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld8(uint32_t taddr, uint32_t* r) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
               : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void bulk_store(void* gdst, uint32_t ssrc, uint32_t bytes, uint64_t pol) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(gdst), "r"(ssrc),
               "r"(bytes), "l"(pol)
               : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void tma_load_2d_hint(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1,
                                                 uint64_t pol) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(dst),
      "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t* r) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),
        "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

template <int EPI, bool OUT_BF16, bool AG = false>
__global__ void __launch_bounds__(AG ? THREADS + AG_THREADS : THREADS, 1)
    gemm_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                const __grid_constant__ Params P) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  __shared__ int64_t s_cn[BN];      // column offsets of the current N-tile (scatter epilogue)
  // split-K over the idle SMs: the fold (t4_xfold_kernel, a programmatic dependent) may be
  // scheduled now; it waits in griddepcontrol.wait for this grid's partials
  if (P.xfold) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  // ring: NST stages of A (16 KB) and B (bn·128 B); EPI 3 keeps 2 stages to leave room for
  // the epilogue's staging buffers (K is short where it is used: CCSD(T) K = 72)
  constexpr int NST = EPI == 3 ? 2 : STAGES;
  const int bn = EPI == 3 ? P.bn : BN;
  const uint32_t b_stage = EPI == 3 ? (uint32_t)P.bn * 128u : (uint32_t)B_BYTES;
  // B-resident mode (EPI 3, P.bres): the whole K extent of the current N-tile's B stays in
  // shared memory while the CTA walks its M-tiles (sched 1 keeps one N-tile for hundreds of
  // consecutive tiles), so only A streams through the ring
  const bool bres = EPI == 3 && P.bres;
  const uint32_t ring = bres ? NST * A_BYTES + P.num_kb * b_stage : NST * (A_BYTES + b_stage);
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sA = smem;
  uint8_t* sB = smem + NST * A_BYTES;
  uint64_t* bars = (uint64_t*)(smem + ring);
  // bars: full[NST], empty[NST], tmem_full[2], tmem_empty[2], b_full, b_empty; then the TMEM slot
  uint32_t* tmem_slot = (uint32_t*)(bars + 2 * NST + 6);
  int64_t* s_koff = (int64_t*)(smem + ring + 256);    // AG: K-chunk offsets
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + NST);
  const uint32_t tfull0 = smem_u32(bars + 2 * NST), tempty0 = smem_u32(bars + 2 * NST + 2);
  const uint32_t bfull = smem_u32(bars + 2 * NST + 4), bempty = smem_u32(bars + 2 * NST + 5);

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&mapA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&mapB) : "memory");
    for (int s = 0; s < NST; ++s) {
      mbar_init(full0 + 8 * s, AG ? 1 + AG_THREADS : 1);    // AG: TMA(B) + every gather thread
      mbar_init(empty0 + 8 * s, 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(tfull0 + 8 * a, 1);
      mbar_init(tempty0 + 8 * a, 256);
    }
    mbar_init(bfull, 1);
    mbar_init(bempty, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ===== TMA producer =====
      const uint64_t pol = policy_evict_last();
      int stage = 0;
      uint32_t phase = 0;
      int b_nb = -1, b_loads = 0;
      for (int u = u_first(P); u < u_last(P); u += u_step(P)) {
        int mb, nb, kb0, kb1, slot;
        u_decode(P, u, &mb, &nb, &kb0, &kb1, &slot);
        const int m0 = mb * BM, n0 = nb * bn;
        if (bres && nb != b_nb) {               // (re)load the resident B of this N-tile
          if (b_loads > 0) mbar_wait(bempty, (b_loads - 1) & 1);
          mbar_expect_tx(bfull, (uint32_t)P.num_kb * b_stage);
          for (int kb = 0; kb < P.num_kb; ++kb)
            tma_load_2d_hint(smem_u32(sB + kb * b_stage), &mapB, bfull, kb * BK, n0, pol);
          b_nb = nb;
          ++b_loads;
        }
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(empty0 + 8 * stage, phase ^ 1);
          const uint32_t fb = full0 + 8 * stage;
          mbar_expect_tx(fb, AG ? b_stage : (bres ? A_BYTES : A_BYTES + b_stage));
          const uint32_t a_dst = smem_u32(sA + stage * A_BYTES), b_dst = smem_u32(sB + stage * b_stage);
          const int k0 = krotate(P, kb, kb0, kb1, mb) * BK;
          if (AG) {
            // A arrives from the gather warps
          } else if (P.a_im2col) {
            int cr[4];
            uint16_t off[2];
            im2col_coords(P, m0, k0, cr, off);
            tma_load_im2col(a_dst, &mapA, fb, cr, off);
          } else if (P.a_box) {               // implicit GEMM: one N-d box {64 k*, …1…, 128 g*}
            int cr[5];
            box_coords(P.abox, m0, k0, cr);
            tma_load_nd(a_dst, &mapA, fb, P.abox.rank, cr);
          } else if (EPI == 3) {       // operands stay in L2 (evict_last) under the output stream
            if (P.a_mn_major) {
              tma_load_2d_hint(a_dst, &mapA, fb, m0, k0, pol);
              tma_load_2d_hint(a_dst + 8192, &mapA, fb, m0 + 64, k0, pol);
            } else {
              tma_load_2d_hint(a_dst, &mapA, fb, k0, m0, pol);
            }
          } else if (P.a_mn_major) {   // box {64 m, 64 k}, two atoms along M
            tma_load_2d(a_dst, &mapA, fb, m0, k0);
            tma_load_2d(a_dst + 8192, &mapA, fb, m0 + 64, k0);
          } else {                     // box {64 k, 128 m}
            tma_load_2d(a_dst, &mapA, fb, k0, m0);
          }
          if (bres) {
            // B is resident
          } else if (EPI == 3) {       // K-major B, box {64 k, bn n}
            tma_load_2d_hint(b_dst, &mapB, fb, k0, n0, pol);
          } else if (P.b_mn_major) {   // box {64 n, 64 k}, four atoms along N
#pragma unroll
            for (int j = 0; j < 4; ++j) tma_load_2d(b_dst + 8192 * j, &mapB, fb, n0 + 64 * j, k0);
          } else {                     // box {64 k, 256 n}
            tma_load_2d(b_dst, &mapB, fb, k0, n0);
          }
          if (++stage == NST) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ===== MMA issuer (one thread) =====
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      int b_nb = -1, b_uses = 0;
      for (int u = u_first(P); u < u_last(P); u += u_step(P), ++it) {
        int mb, nb, kb0, kb1, slot;
        u_decode(P, u, &mb, &nb, &kb0, &kb1, &slot);
        const int acc = it & 1;
        if (bres && nb != b_nb) {
          if (b_uses > 0) mma_commit(bempty);   // the old B is free once the MMAs issued so far retire
          mbar_wait(bfull, b_uses & 1);
          b_nb = nb;
          ++b_uses;
        }
        mbar_wait(tempty0 + 8 * acc, ((it >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t d = tmem + acc * BN;
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(full0 + 8 * stage, phase);
          tc_fence_after();
          const uint32_t a0 = smem_u32(sA + stage * A_BYTES),
                         b0 = smem_u32(sB + (bres ? kb : stage) * b_stage);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            // K-major: +32 B per 16-element K step inside the 128-B swizzled row;
            // MN-major: +16 rows × 128 B = 2048 B per K step (LBO = next 64-wide MN atom)
            const uint64_t ad = P.a_mn_major ? sdesc(a0 + 2048 * k, 8192, 1024) : sdesc(a0 + 32 * k, 16, 1024);
            const uint64_t bd = P.b_mn_major ? sdesc(b0 + 2048 * k, 8192, 1024) : sdesc(b0 + 32 * k, 16, 1024);
            mma_bf16(d, ad, bd, P.idesc, kb != kb0 || k != 0);
          }
          mma_commit(empty0 + 8 * stage);            // smem stage free once these MMAs retire
          if (++stage == NST) { stage = 0; phase ^= 1; }
        }
        mma_commit(tfull0 + 8 * acc);                 // accumulator ready for the epilogue
      }
    }
  } else if (AG && warp >= THREADS / 32) {
    // ===== A gather producer (warps 10..13): the A tile straight from the operand through
    // its row / K-chunk offset tables with 16-byte cp.async into the SWIZZLE_128B K-major
    // layout TMA would produce (16-B chunk c of row r at (c ^ (r & 7)) * 16), so no
    // materialised im2col / permuted copy.  Thread → K chunk (gt & 7) of rows gt/8 + 16 i.
    // A stage is published AG_LAG k-blocks later: wait_group, proxy fence, arrive.
    const int gt = threadIdx.x - THREADS;
    const int run = P.ag4 ? 4 : 8;
    for (int i = gt; i < P.nkc; i += AG_THREADS) s_koff[i] = __ldg(P.aK + run * (int64_t)i);
    named_sync(2, AG_THREADS);
    if (P.ag4) {
      // 8-byte variant (K offsets contiguous only in runs of 4, e.g. MCC_Caps' l): thread →
      // half-chunk (gt & 15) of rows gt/16 + 8 i; half h of 16-B chunk c of row r at
      // ((c ^ (r & 7)) * 16 + 8 h)
      const int hc = gt & 15, rb4 = gt >> 4;
      int stage = 0;
      uint32_t phase = 0;
      int g = 0;
      for (int u = u_first(P); u < u_last(P); u += u_step(P)) {
        int mb, nb, kb0, kb1, slot;
        u_decode(P, u, &mb, &nb, &kb0, &kb1, &slot);
        const int64_t m0 = (int64_t)mb * BM;
        int64_t ro[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          const int64_t m = m0 + rb4 + 8 * i;
          ro[i] = m < P.M ? __ldg(P.aM + m) : -1;
        }
        for (int kb = kb0; kb < kb1; ++kb, ++g) {
          mbar_wait(empty0 + 8 * stage, phase ^ 1);
          const uint32_t base = smem_u32(sA + stage * A_BYTES);
          const int kc = krotate(P, kb, kb0, kb1, (int)mb) * (BK / 4) + hc;
          const int64_t ko = kc < P.nkc ? s_koff[kc] : -1;
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            const int r = rb4 + 8 * i;
            const uint32_t dst = base + r * 128 + (((hc >> 1) ^ (r & 7)) << 4) + ((hc & 1) << 3);
            if (ro[i] >= 0 && ko >= 0)
              asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(dst), "l"(P.Ag + ro[i] + ko) : "memory");
            else asm volatile("st.shared.v2.u32 [%0], {%1, %1};" ::"r"(dst), "r"(0) : "memory");
          }
          cp_async_commit();
          if (g >= P.ag_lag) {
            if (P.ag_lag == 1) cp_async_wait<1>();
            else if (P.ag_lag == 2) cp_async_wait<2>();
            else cp_async_wait<3>();
            fence_proxy_async();
            mbar_arrive(full0 + 8 * ((g - P.ag_lag) % NST));
          }
          if (++stage == NST) { stage = 0; phase ^= 1; }
        }
      }
      cp_async_wait<0>();
      fence_proxy_async();
      for (int j = g - P.ag_lag < 0 ? 0 : g - P.ag_lag; j < g; ++j) mbar_arrive(full0 + 8 * (j % NST));
    } else {
    const int ch = gt & 7, rb = gt >> 3;
    int stage = 0;
    uint32_t phase = 0;
    int g = 0;                                   // k-blocks issued so far
    for (int u = u_first(P); u < u_last(P); u += u_step(P)) {
      int mb, nb, kb0, kb1, slot;
      u_decode(P, u, &mb, &nb, &kb0, &kb1, &slot);
      const int64_t m0 = (int64_t)mb * BM;
      int64_t ro[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int64_t m = m0 + rb + 16 * i;
        ro[i] = m < P.M ? __ldg(P.aM + m) : -1;
      }
      for (int kb = kb0; kb < kb1; ++kb, ++g) {
        mbar_wait(empty0 + 8 * stage, phase ^ 1);
        const uint32_t base = smem_u32(sA + stage * A_BYTES);
        const int kc = krotate(P, kb, kb0, kb1, (int)mb) * (BK / 8) + ch;
        const int64_t ko = kc < P.nkc ? s_koff[kc] : -1;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int r = rb + 16 * i;
          const uint32_t dst = base + r * 128 + ((ch ^ (r & 7)) << 4);
          if (ro[i] >= 0 && ko >= 0) cp_async16(dst, P.Ag + ro[i] + ko);
          else asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(dst), "r"(0) : "memory");
        }
        cp_async_commit();
        if (g >= P.ag_lag) {
          if (P.ag_lag == 1) cp_async_wait<1>();
          else if (P.ag_lag == 2) cp_async_wait<2>();
          else cp_async_wait<3>();
          fence_proxy_async();
          mbar_arrive(full0 + 8 * ((g - P.ag_lag) % NST));
        }
        if (++stage == NST) { stage = 0; phase ^= 1; }
      }
    }
    cp_async_wait<0>();
    fence_proxy_async();
    for (int j = g - P.ag_lag < 0 ? 0 : g - P.ag_lag; j < g; ++j) mbar_arrive(full0 + 8 * (j % NST));
    }
  } else if (EPI == 3) {
    // ===== bulk-run epilogue: the output is contiguous along n in runs of L = bn/2 and a
    // warp owns 32 accumulator rows × one run.  TMEM → registers → this warp's staging
    // buffer in output order [row][L]; then the rows whose offsets continue each other
    // (cM[m+1] = cM[m] + L, e.g. CCSD(T)'s p5) leave as ONE cp.async.bulk store of
    // rows·L·4 bytes (measured 6.8-7.2 TB/s for 36-72 KB pieces vs 4.1-5.1 TB/s for
    // per-thread stores of the same layout, tools/wbw_probe.cu).  Double-buffered
    // staging: a buffer is rewritten only after its previous bulk read completed. =====
    const int quad = warp & 3;
    const int half = (warp - 2) >> 2;
    const int L = bn >> 1;
    const int row = quad * 32 + lane;
    float* stg0 = (float*)(smem + ring + 1024) + (size_t)(warp - 2) * P.nstg * 32 * L;
    int it = 0, sb = 0;
    int cached_nb = -1;
    const uint64_t pol = policy_evict_first();
    // the row offset cM[m] of the NEXT tile is loaded one iteration ahead (its L2 latency
    // was the epilogue's largest stall)
    auto row_off = [&](int u) -> int64_t {
      if (u >= u_last(P)) return -1;
      int mb, nbk, kb0, kb1, slot;
      u_decode(P, u, &mb, &nbk, &kb0, &kb1, &slot);
      const int64_t m = (int64_t)mb * BM + row;
      return m < P.M ? P.cbase + __ldg(P.cM + m) : -1;
    };
    int64_t crow_next = row_off(u_first(P));
    for (int u = u_first(P); u < u_last(P); u += u_step(P), ++it) {
      const int acc = it & 1;
      int mb, nbk, kb0, kb1, slot;
      u_decode(P, u, &mb, &nbk, &kb0, &kb1, &slot);
      const int64_t crow_cur = crow_next;
      crow_next = row_off(u + u_step(P));
      if (nbk != cached_nb) {
        const int et = threadIdx.x - 64;
        named_sync(1, 256);
        const int64_t nn = (int64_t)nbk * bn + et;
        if (et < bn) s_cn[et] = __ldg(P.cN + min(nn, P.N - 1));
        named_sync(1, 256);
        cached_nb = nbk;
      }
      const bool mok = crow_cur >= 0;
      const int64_t crow = mok ? crow_cur : 0;
      const bool nok = (int64_t)nbk * bn + half * L < P.N;
      float* stg = stg0 + sb * 32 * L;
      if (lane == 0) {
        if (P.nstg == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
        else asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      }
      __syncwarp();
      mbar_wait(tfull0 + 8 * acc, (it >> 1) & 1);
      tc_fence_after();
      const uint32_t tbase = tmem + ((uint32_t)(quad * 32) << 16) + acc * BN + half * L;
      // 16 columns per batch of two x8 loads (one wait), then 16-byte st.shared in pairs of
      // chunks; lanes with bit 2 set take the pair in the other order, which makes each
      // 8-lane phase hit 8 distinct bank groups (row pitch L·4 B ≡ 2 groups mod 8 for L = 72)
      const uint32_t srow = smem_u32(stg + lane * L);
      const bool flip = P.e3flip && ((lane >> 2) & 1);
#pragma unroll 1
      for (int c = 0; c < L; c += 16) {
        uint32_t r[16];
        tmem_ld8(tbase + c, r);
        if (c + 8 < L) tmem_ld8(tbase + c + 8, r + 8);
        tmem_wait_ld();
#pragma unroll
        for (int h = 0; h < 16; h += 8) {
          if (c + h < L) {
            uint32_t v[8];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              v[j] = flip ? r[h + 4 + j] : r[h + j];
              v[4 + j] = flip ? r[h + j] : r[h + 4 + j];
            }
            const uint32_t a0 = srow + 4 * (c + h + (flip ? 4 : 0)), a1 = srow + 4 * (c + h + (flip ? 0 : 4));
            asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a0), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3])
                         : "memory");
            asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a1), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
                         : "memory");
          }
        }
      }
      tc_fence_before();
      mbar_arrive(tempty0 + 8 * acc);          // accumulator free for the MMA of tile it+2
      fence_proxy_async();
      __syncwarp();
      // row pieces: a piece starts where the output offset does not continue the previous row
      const int64_t prev = __shfl_up_sync(0xffffffffu, crow, 1);
      const bool start = mok && (lane == 0 || crow != prev + L);
      unsigned st = __ballot_sync(0xffffffffu, start);
      const int nvalid = __popc(__ballot_sync(0xffffffffu, mok));
      if (!nok) st = 0;
      const int64_t coff = s_cn[half * L];
      while (st) {
        const int s0 = __ffs(st) - 1;
        st &= st - 1;
        const int e0 = st ? __ffs(st) - 1 : nvalid;
        const int64_t cs = __shfl_sync(0xffffffffu, crow, s0);
        if (lane == 0) bulk_store(P.C + cs + coff, smem_u32(stg + s0 * L), (uint32_t)((e0 - s0) * L * 4), pol);
      }
      if (lane == 0) asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      if (P.nstg == 2) sb ^= 1;
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    __syncwarp();
  } else {
    // ===== epilogue: warps 2..9; warp → TMEM lane quadrant (warp % 4) and a half of the
    // 256 accumulator columns (two warps per sub-partition hide the store latency) =====
    const int quad = warp & 3;
    const int half = (warp - 2) >> 2;
    const int row = quad * 32 + lane;
    int it = 0;
    int cached_nb = -1;
    for (int u = u_first(P); u < u_last(P); u += u_step(P), ++it) {
      const int acc = it & 1;
      int mb, nbk, kb0, kb1, slot;
      u_decode(P, u, &mb, &nbk, &kb0, &kb1, &slot);
      const int64_t m = (int64_t)mb * BM + row;
      const int64_t n0 = (int64_t)nbk * BN + half * (BN / 2);
      if (EPI >= 1 && nbk != cached_nb) {
        // (re)load this N-tile's column offsets into shared memory (epilogue warps only)
        const int et = threadIdx.x - 64;
        named_sync(1, 256);
        const int64_t nn = (int64_t)nbk * BN + et;
        s_cn[et] = __ldg(P.cN + min(nn, P.N - 1));
        named_sync(1, 256);
        cached_nb = nbk;
      }
      mbar_wait(tfull0 + 8 * acc, (it >> 1) & 1);
      tc_fence_after();
      const bool mok = m < P.M;
      const int64_t crow = P.cbase + (EPI == 0 ? (mok ? m : 0) * P.ldc : __ldg(P.cM + (mok ? m : 0)));
      // split-K tail (as in gemm2_kernel): splits 0..S-2 write a dense fp32 partial tile
      // [128][256] and count their 8 warps in; the last split waits for them and folds
      // p_0 + … + p_{S-2} + own in split order before the store
      const bool split = slot >= 0;
      const int ti = split ? slot / P.ssplit : 0;
      const bool last = split && !P.xfold && slot % P.ssplit == P.ssplit - 1;
      unsigned* cnt = P.tail_cnt + 2 * ti;
      const int64_t prel = (int64_t)row * BN + half * (BN / 2);
      float* prow = (split && !last) ? P.part + (int64_t)slot * (BM * BN) + prel : nullptr;
      if (last) {
        if (lane == 0)
          while (*((volatile unsigned*)cnt) < 8u * (unsigned)(P.ssplit - 1)) __nanosleep(64);
        __syncwarp();
        __threadfence();
      }
#pragma unroll 1
      for (int c = 0; c < BN / 64; ++c) {
        uint32_t r[32];
        tmem_ld32(tmem + ((uint32_t)(quad * 32) << 16) + acc * BN + half * (BN / 2) + c * 32, r);
        const int64_t nb = n0 + c * 32;
        if (last) {
          const float* p0 = P.part + (int64_t)(ti * P.ssplit) * (BM * BN) + prel + c * 32;
#pragma unroll
          for (int j4 = 0; j4 < 8; ++j4) {
            float4 a = *reinterpret_cast<const float4*>(p0 + 4 * j4);
            for (int s2 = 1; s2 < P.ssplit - 1; ++s2) {
              const float4 b = *reinterpret_cast<const float4*>(p0 + (int64_t)s2 * (BM * BN) + 4 * j4);
              a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
            }
            r[4 * j4] = __float_as_uint(a.x + __uint_as_float(r[4 * j4]));
            r[4 * j4 + 1] = __float_as_uint(a.y + __uint_as_float(r[4 * j4 + 1]));
            r[4 * j4 + 2] = __float_as_uint(a.z + __uint_as_float(r[4 * j4 + 2]));
            r[4 * j4 + 3] = __float_as_uint(a.w + __uint_as_float(r[4 * j4 + 3]));
          }
        }
        if (prow) {
          float4* dst = reinterpret_cast<float4*>(prow + c * 32);
#pragma unroll
          for (int j = 0; j < 8; ++j)
            dst[j] = make_float4(__uint_as_float(r[4 * j]), __uint_as_float(r[4 * j + 1]), __uint_as_float(r[4 * j + 2]),
                                 __uint_as_float(r[4 * j + 3]));
        } else if (EPI == 0) {
          // row-major fp32 C: each thread writes 128 contiguous bytes of its row
          if (mok && nb + 32 <= P.N && ((crow + nb) & 3) == 0) {
            float4* dst = reinterpret_cast<float4*>(P.C + crow + nb);
#pragma unroll
            for (int j = 0; j < 8; ++j)
              dst[j] = make_float4(__uint_as_float(r[4 * j]), __uint_as_float(r[4 * j + 1]),
                                   __uint_as_float(r[4 * j + 2]), __uint_as_float(r[4 * j + 3]));
          } else if (mok) {
#pragma unroll
            for (int j = 0; j < 32; ++j)
              if (nb + j < P.N) P.C[crow + nb + j] = __uint_as_float(r[j]);
          }
        } else if (EPI == 2) {
          // run-8 scatter: the output is contiguous along n in aligned runs of 8 (the plan
          // checked cN and the alignment), so each thread stores its row's 32 columns as
          // four 32-byte vectors (STG.256; 16 B for bf16) at crow + cN[run start]
          if (mok && P.run4 && !OUT_BF16) {
            // run-4: eight 16-byte vectors at crow + cN[run start]
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              if (nb + 4 * j < P.N) {
                const int64_t o = crow + s_cn[half * (BN / 2) + c * 32 + 4 * j];
                const uint32_t* v = r + 4 * j;
                asm volatile("st.global.cs.v4.b32 [%0], {%1, %2, %3, %4};" ::"l"(P.C + o), "r"(v[0]), "r"(v[1]), "r"(v[2]),
                             "r"(v[3])
                             : "memory");
              }
            }
          } else if (mok) {
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              if (nb + 8 * j < P.N) {
                const int64_t o = crow + s_cn[half * (BN / 2) + c * 32 + 8 * j];
                const uint32_t* v = r + 8 * j;
                if (OUT_BF16) {
                  uint32_t h[4];
#pragma unroll
                  for (int q = 0; q < 4; ++q) {
                    const __nv_bfloat162 t = __floats2bfloat162_rn(__uint_as_float(v[2 * q]), __uint_as_float(v[2 * q + 1]));
                    h[q] = *reinterpret_cast<const uint32_t*>(&t);
                  }
                  asm volatile("st.global.cs.v4.b32 [%0], {%1, %2, %3, %4};" ::"l"((__nv_bfloat16*)P.C + o), "r"(h[0]),
                               "r"(h[1]), "r"(h[2]), "r"(h[3])
                               : "memory");
                } else {
                  asm volatile("st.global.cs.v8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(P.C + o), "r"(v[0]),
                               "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
                               : "memory");
                }
              }
            }
          }
        } else {
          // scatter through the output tables: column offsets first (branch-free,
          // clamped read-only loads), then the stores; lanes = consecutive rows, so a
          // store instruction is coalesced when the output is contiguous along m
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            int64_t co[16];
#pragma unroll
            for (int j = 0; j < 16; ++j) co[j] = s_cn[half * (BN / 2) + c * 32 + h * 16 + j];
#pragma unroll
            for (int j = 0; j < 16; ++j) {
              if (mok && nb + h * 16 + j < P.N) {
                const int64_t o = crow + co[j];
                const float v = __uint_as_float(r[h * 16 + j]);
                if (OUT_BF16) ((__nv_bfloat16*)P.C)[o] = __float2bfloat16_rn(v);
                else __stcs(P.C + o, v);
              }
            }
          }
        }
      }
      if (split && !last && !P.xfold) {   // publish this warp's part of the partial tile
        __threadfence();
        __syncwarp();
        if (lane == 0) atomicAdd(cnt, 1u);
      } else if (last) {               // 8 warps leave; the last one resets the counters
        __syncwarp();
        if (lane == 0 && atomicAdd(cnt + 1, 1u) == 7u) {
          cnt[0] = 0u;
          cnt[1] = 0u;
        }
      }
      tc_fence_before();
      mbar_arrive(tempty0 + 8 * acc);
    }
  }
  __syncwarp();                  // lanes 1..31 of warps 0/1 wait for their role lane
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS));
  }
}

// ---- 2-SM variant: a CTA pair (cluster 2×1) computes a 256×256 tile with
// tcgen05.mma.cta_group::2 (M = 256 split over the two SMs' TMEM, each SM staging half of A
// and half of B), so each SM streams 32 KB instead of 48 KB of operands per 64-deep k-block
// for the same MMA work.  Barriers: the leader's full barrier counts both producers and
// both CTAs' TMA bytes (cta_group::2 TMA signals the leader); MMA commits are multicast to
// both CTAs' empty / tmem-full barriers; both epilogues release the accumulator at the
// leader's tmem-empty barrier.
// Work schedule of a CTA pair: data-parallel whole tiles u = pair, pair + npairs, … < nfull,
// then the pair's stream-K range [s_p, s_{p+1}), s_p = p·sk_w / sk_pairs, cut at tile
// boundaries into segments (tile, kb0, kb1).  Role of a segment: 0 whole tile; 1 producer
// (kb0 > 0: the partial sum goes to the pair's workspace slot — it is always the pair's
// FIRST stream-K segment); 2 finisher (kb0 = 0, kb1 < num_kb: the pair's LAST segment; it
// adds the producers' partials p+1, p+2, … in k order before the store).  Producers run
// first and finishers last, so a finisher finds its partials (nearly always) published;
// all pairs are co-resident (persistent grid), so the flag waits cannot deadlock.
struct SkWork { int t, kb0, kb1, role, u0, nu; };   // u0 / nu: first column unit and units (vmode)
template <bool LEAN = false>
struct SkIter {
  int u, step, nfull, kb, ups, tiles_n;
  bool vmode;
  int64_t k, e;
  __device__ __forceinline__ SkIter(const Params& P, int pair, int npairs) {
    u = pair;
    step = npairs;
    nfull = P.nfull;
    kb = P.num_kb;
    vmode = !LEAN && P.vmode != 0;
    ups = P.ups;
    tiles_n = P.tiles_n;
    k = e = 0;
    if (vmode) {                     // column units after the nfull whole 256×512 tiles
      const int64_t g0 = nfull > 0 ? (int64_t)(nfull / tiles_n) * ups + 4 * (nfull % tiles_n) : 0;
      k = g0 + (int64_t)pair * (P.vunits - g0) / npairs;
      e = g0 + (int64_t)(pair + 1) * (P.vunits - g0) / npairs;
    } else if (!LEAN && P.sk_pairs > 0 && pair < P.sk_pairs) {
      k = (int64_t)pair * P.sk_w / P.sk_pairs;
      e = (int64_t)(pair + 1) * P.sk_w / P.sk_pairs;
    }
  }
  __device__ __forceinline__ bool next(SkWork* w) {
    w->u0 = 0;
    w->nu = 0;
    if (vmode) {                     // whole tiles, then units k … e-1: strip k / ups, ≤ 4 units per tile
      if (u < nfull) {
        const int cu = 4 * (u % tiles_n);
        w->t = u / tiles_n; w->kb0 = 0; w->kb1 = kb; w->role = 0; w->u0 = cu; w->nu = min(4, ups - cu);
        u += step;
        return true;
      }
      if (k >= e) return false;
      const int strip = (int)(k / ups), cu = (int)(k % ups);
      const int nu = (int)min((int64_t)4, min(e - k, (int64_t)(ups - cu)));
      w->t = strip; w->kb0 = 0; w->kb1 = kb; w->role = 0; w->u0 = cu; w->nu = nu;
      k += nu;
      return true;
    }
    if (u < nfull) {
      w->t = u; w->kb0 = 0; w->kb1 = kb; w->role = 0;
      u += step;
      return true;
    }
    if (LEAN || k >= e) return false;
    const int64_t x = k / kb;
    w->t = nfull + (int)x;
    w->kb0 = (int)(k - x * kb);
    const int64_t rem = e - k;
    w->kb1 = rem < (int64_t)(kb - w->kb0) ? w->kb0 + (int)rem : kb;
    w->role = (w->kb0 == 0 && w->kb1 == kb) ? 0 : (w->kb0 == 0 ? 2 : 1);
    k += w->kb1 - w->kb0;
    return true;
  }
};

constexpr int S2 = 5;                          // stages (32 KB each)
constexpr int A2_BYTES = 128 * BK * 2;         // this CTA's half of A (16 KB)
constexpr int B2_BYTES = 128 * BK * 2;         // this CTA's half of B (16 KB)
constexpr int STAGE2_BYTES = A2_BYTES + B2_BYTES;
constexpr int STG2_BYTES = 2 * 8 * 32 * 32 * 4;  // epilogue staging: 2 × 32×32 fp32 per epilogue warp
constexpr int S2W = 3;                         // stages of the wide (NW = 512) ring (48 KB each)
constexpr int SMEM2_BYTES = S2 * STAGE2_BYTES + 1024 + 1024 + STG2_BYTES;   // ring, align slack, barriers, staging
static_assert(S2W * (A2_BYTES + 2 * B2_BYTES) <= S2 * STAGE2_BYTES, "wide ring must fit the 2-SM smem budget");
static_assert(SMEM2_BYTES <= 232448, "2-SM kernel exceeds 227 KB of shared memory");

__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t map_to_rank(uint32_t addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
  return r;
}
__device__ __forceinline__ uint32_t map_to_rank0(uint32_t addr) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(r) : "r"(addr));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void tma_load_2d_cg2(uint32_t dst, const CUtensorMap* map, uint32_t bar_cluster, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"((uint64_t)map), "r"(bar_cluster), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tma_load_im2col_cg2(uint32_t dst, const CUtensorMap* map, uint32_t bar_cluster, const int* c,
                                                    const uint16_t* off) {
  asm volatile(
      "cp.async.bulk.tensor.4d.im2col.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};" ::"r"(dst),
      "l"((uint64_t)map), "r"(bar_cluster), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]), "h"(off[0]), "h"(off[1])
      : "memory");
}
__device__ __forceinline__ void mma_bf16_cg2(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
// the same MMA keeping its A operand in the tensor core's collector buffer (A_KEEP) for the
// next MMA, which reads it from there (A_REUSE) instead of from shared memory
__device__ __forceinline__ void mma_bf16_cg2_afill(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16.collector::a::fill [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void mma_bf16_cg2_alast(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16.collector::a::lastuse [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
// commit to the barrier at `bar`'s offset in every CTA of `mask` (cluster ranks)
__device__ __forceinline__ void mma_commit_cg2_mask(uint32_t bar, uint16_t mask) {
  asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(bar),
               "h"(mask)
               : "memory");
}
// B piece multicast to the CTAs of `mask`; with cta_group::2 the complete_tx of every
// destination lands on the barrier at bar's offset in that destination's pair leader
__device__ __forceinline__ void tma_load_2d_cg2_mc(uint32_t dst, const CUtensorMap* map, uint32_t bar_cluster, int c0, int c1,
                                                   uint16_t mask) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(dst),
      "l"((uint64_t)map), "r"(bar_cluster), "r"(c0), "r"(c1), "h"(mask)
      : "memory");
}
// TMA tensor store of a 32×32 fp32 box (128B-swizzled smem image) at {n, m}; OOB clipped
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"((uint64_t)map), "r"(src),
               "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void mma_commit_cg2(uint32_t bar) {
  asm volatile(
      "{\n\t.reg .b16 m;\n\tmov.b16 m, 3;\n\t"
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], m;\n\t}" ::"r"(bar)
      : "memory");
}
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t bar_cluster) {
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(bar_cluster) : "memory");
}
// CL = 2: one CTA pair per cluster.  CL = 4: two pairs (cluster ranks {0,1} and {2,3}) on
// vertically adjacent 256×256 tiles of one 512×256 super-tile; they share the B tile, each
// CTA loading half of its B half (8 KB) by TMA multicast into both pairs, so a CTA reads
// 24 KB instead of 32 KB from L2 per k-block.  Stage slots are freed by the commits of
// both pairs (empty barriers count 2, commit mask 0xF).
//
// NW = 512 (wide tiles, CL = 2): a pair owns a 256×512 tile as two N=256 MMAs per k-step
// into TMEM columns [0,256) and [256,512) — all 512 columns, so there is one accumulator:
// the epilogue drains column half 0, frees it (tempty[0]), then half 1 (tempty[1]), and the
// next tile's first MMAs into half h wait only for tempty[h].  Per k-block a CTA loads its
// A half once for twice the MMA work (A 16 + B 32 KB per 8.4 MFLOP instead of 16 + 16 per
// 4.2): A — the im2col operand of a convolution — is requested half as often.
// WST (wide tiles only): ring stages — 3 with double-buffered epilogue staging, or 4 with
// single-buffered staging (4 × 48 KB + 32 KB fits the 227 KB budget; tile knob stages=4:
// MCC conv5_1 +1-3 %, MatMul 4096³ / 8192³ -2 / -3 %: the single staging buffer slows the
// whole-tile epilogues)
template <bool OUT_ROWMAJOR, int CL, int NW = 256, int WST = S2W, bool LEAN = false>
__global__ void __cluster_dims__(CL, 1, 1) __launch_bounds__(THREADS, 1)
    gemm2_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                 const __grid_constant__ CUtensorMap mapC, const __grid_constant__ Params P) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // LEAN: whole tiles only (no stream-K roles, no column units, no trace) — a smaller
  // instance whose hot loops share the instruction cache with less cold code
  unsigned long long* const trace = LEAN ? nullptr : P.trace;
  const bool vm = !LEAN && P.vmode != 0;
  constexpr int NH = NW / 256;                   // N=256 MMAs per k-step
  constexpr int NS = NW == 512 ? WST : S2;       // ring stages
  constexpr int EPB = (NW == 512 && WST == 4) ? 1 : 2;   // epilogue staging buffers per warp
  static_assert(NW != 512 || WST * (A2_BYTES + 2 * B2_BYTES) + 2048 + EPB * 8 * 4096 <= 232448, "smem budget");
  constexpr int BSTG = NH * B2_BYTES;            // this CTA's B bytes per stage
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sA = smem;
  uint8_t* sB = smem + NS * A2_BYTES;
  uint64_t* bars = (uint64_t*)(smem + NS * (A2_BYTES + BSTG));
  uint32_t* tmem_slot = (uint32_t*)(bars + 2 * NS + 4);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t crank = cluster_rank();
  const uint32_t pp = crank >> 1;                // pair within the cluster
  const uint32_t rank = crank & 1;               // CTA within the pair
  const bool leader = rank == 0;
  constexpr int NPP = CL / 2;                    // pairs per cluster
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + NS);
  const uint32_t tfull0 = smem_u32(bars + 2 * NS), tempty0 = smem_u32(bars + 2 * NS + 2);
  // pair tiles: tiles_m/tiles_n count 256×NW tiles; clusters stride over them
  const int cluster_id = blockIdx.x / CL, nclusters = gridDim.x / CL;
  const int pair_gid = cluster_id * NPP + (int)pp;   // partial slot / trace row of this pair
  if (trace && threadIdx.x == 0 && pair_gid < 256) trace[8 * P.trace_n + 2 * pair_gid + rank * 512] = gtimer();

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&mapA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&mapB) : "memory");
    if (P.c_vec4) asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&mapC) : "memory");
    for (int s = 0; s < NS; ++s) {
      mbar_init(full0 + 8 * s, 2);
      mbar_init(empty0 + 8 * s, NPP);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(tfull0 + 8 * a, 1);
      mbar_init(tempty0 + 8 * a, 16);          // 8 epilogue warps × 2 CTAs
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  tc_fence_before();
  cluster_sync_all();
  __syncthreads();               // (also orders the TMEM-address slot for racecheck)
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ===== TMA producer (both CTAs; bytes are counted at the leader's full barrier) =====
      int stage = 0;
      uint32_t phase = 0;
      SkIter<LEAN> wi(P, cluster_id, nclusters);
      SkWork w;
      while (wi.next(&w)) {
        const int t = w.t, kb0 = w.kb0, kb1 = w.kb1;
        const int m0 = vm ? t * 256 + (int)rank * 128 : ((t / P.tiles_n) * NPP + (int)pp) * 256 + (int)rank * 128;
        const int n0 = vm ? 128 * w.u0 + (int)rank * 128 : (t % P.tiles_n) * NW + (int)rank * 128;
        // vmode: MMA h covers units u0+2h, u0+2h+1 (N = 256, 128 columns per CTA) or only the
        // tile's odd last unit (N = 128, 64 columns per CTA: one 64-column MN-major box)
        const int vnh = (w.nu + 1) / 2;
        const bool vodd = (w.nu & 1) != 0;
        const uint32_t bbytes = !vm ? (uint32_t)BSTG
                                         : (uint32_t)(vnh * B2_BYTES - (vodd && P.b_mn_major ? B2_BYTES / 2 : 0));
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(empty0 + 8 * stage, phase ^ 1);
          const uint32_t fb_leader = map_to_rank(full0 + 8 * stage, 2 * pp);
          if (leader) mbar_expect_tx(full0 + 8 * stage, 2 * (A2_BYTES + bbytes));
          else mbar_arrive_cluster(fb_leader);
          const uint32_t a_dst = smem_u32(sA + stage * A2_BYTES), b_dst = smem_u32(sB + stage * BSTG);
          const int k0 = krotate(P, kb, kb0, kb1, t / P.tiles_n) * BK;
          if (P.a_im2col) {
            int cr[4];
            uint16_t off[2];
            im2col_coords(P, m0, k0, cr, off);
            tma_load_im2col_cg2(a_dst, &mapA, fb_leader, cr, off);
          } else if (P.a_mn_major) {
            tma_load_2d_cg2(a_dst, &mapA, fb_leader, m0, k0);
            tma_load_2d_cg2(a_dst + 8192, &mapA, fb_leader, m0 + 64, k0);
          } else {
            tma_load_2d_cg2(a_dst, &mapA, fb_leader, k0, m0);
          }
          if (CL == 4) {               // this pair's 64-row piece of the B half, to both pairs
            const uint16_t mask = (uint16_t)((1u << rank) | (1u << (2 + rank)));
            if (P.b_mn_major) tma_load_2d_cg2_mc(b_dst + pp * 8192, &mapB, fb_leader, n0 + 64 * pp, k0, mask);
            else tma_load_2d_cg2_mc(b_dst + pp * 8192, &mapB, fb_leader, k0, n0 + 64 * pp, mask);
          } else if (vm) {
            for (int h = 0; h < vnh; ++h) {
              const bool half_unit = vodd && h == vnh - 1;     // N = 128: 64 columns per CTA
              const int nb = half_unit ? 128 * (w.u0 + 2 * h) + (int)rank * 64 : n0 + 256 * h;
              if (P.b_mn_major) {
                tma_load_2d_cg2(b_dst + h * B2_BYTES, &mapB, fb_leader, nb, k0);
                if (!half_unit) tma_load_2d_cg2(b_dst + h * B2_BYTES + 8192, &mapB, fb_leader, nb + 64, k0);
              } else {
                tma_load_2d_cg2(b_dst + h * B2_BYTES, &mapB, fb_leader, k0, nb);
              }
            }
          } else {
#pragma unroll
            for (int h = 0; h < NH; ++h) {   // B piece h: columns 256h + 128·rank + [0, 128)
              if (P.b_mn_major) {
                tma_load_2d_cg2(b_dst + h * B2_BYTES, &mapB, fb_leader, n0 + 256 * h, k0);
                tma_load_2d_cg2(b_dst + h * B2_BYTES + 8192, &mapB, fb_leader, n0 + 256 * h + 64, k0);
              } else {
                tma_load_2d_cg2(b_dst + h * B2_BYTES, &mapB, fb_leader, k0, n0 + 256 * h);
              }
            }
          }
          if (++stage == NS) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && leader) {
      // ===== MMA issuer: leader CTA only, one thread, M=256 × N=256 per instruction =====
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      SkIter<LEAN> wi(P, cluster_id, nclusters);
      SkWork w;
      for (; wi.next(&w); ++it) {
        const int u = it;
        const int kb0 = w.kb0, kb1 = w.kb1;
        const int acc = NH == 1 ? it & 1 : 0;
        const long long ct0 = trace ? clock64() : 0;
        if (NH == 1) {
          mbar_wait(tempty0 + 8 * acc, ((it >> 1) & 1) ^ 1);
          if (trace && pair_gid + u * nclusters * NPP < P.trace_n)
            trace[8 * (pair_gid + u * nclusters * NPP) + 5] = (unsigned long long)(clock64() - ct0);
          tc_fence_after();
        }
        const uint32_t d = tmem + acc * BN;
        long long wfull = 0, cfirst = 0;
        for (int kb = kb0; kb < kb1; ++kb) {
          if (trace && kb == kb0) cfirst = clock64();
          if (trace) {
            const long long c0 = clock64();
            mbar_wait(full0 + 8 * stage, phase);
            wfull += clock64() - c0;
          } else {
            mbar_wait(full0 + 8 * stage, phase);
          }
          tc_fence_after();
          if (trace && kb == kb0 && pair_gid + u * nclusters * NPP < P.trace_n) {
            trace[8 * (pair_gid + u * nclusters * NPP)] = ((unsigned long long)smid() << 32) | (unsigned)pair_gid;
            trace[8 * (pair_gid + u * nclusters * NPP) + 1] = gtimer();
          }
          const uint32_t a0 = smem_u32(sA + stage * A2_BYTES), b0 = smem_u32(sB + stage * BSTG);
          const int mnh = vm ? (w.nu + 1) / 2 : NH;
          if (NH == 2 && P.areuse && mnh == 2) {
            // k-outer: the two column halves' MMAs of one 16-deep k slice share A, read from
            // shared memory once (collector fill) and reused by the second MMA
            if (kb == kb0) {
#pragma unroll
              for (int h = 0; h < 2; ++h) {
                const long long ch = trace ? clock64() : 0;
                mbar_wait(tempty0 + 8 * h, (it & 1) ^ 1);
                if (trace && pair_gid + u * nclusters * NPP < P.trace_n)
                  trace[8 * (pair_gid + u * nclusters * NPP) + 5] += (unsigned long long)(clock64() - ch);
              }
              tc_fence_after();
            }
#pragma unroll
            for (int k = 0; k < BK / 16; ++k) {
              const uint64_t ad = P.a_mn_major ? sdesc(a0 + 2048 * k, 8192, 1024) : sdesc(a0 + 32 * k, 16, 1024);
              const uint64_t bd0 = P.b_mn_major ? sdesc(b0 + 2048 * k, 8192, 1024) : sdesc(b0 + 32 * k, 16, 1024);
              const uint64_t bd1 = P.b_mn_major ? sdesc(b0 + B2_BYTES + 2048 * k, 8192, 1024)
                                                : sdesc(b0 + B2_BYTES + 32 * k, 16, 1024);
              const uint32_t accf = (kb != kb0) || k != 0;
              mma_bf16_cg2_afill(d, ad, bd0, P.idesc, accf);
              mma_bf16_cg2_alast(d + 256, ad, bd1, (vm && (w.nu & 1)) ? P.idesc128 : P.idesc, accf);
            }
          } else
#pragma unroll
          for (int h = 0; h < NH; ++h) {
            if (h >= mnh) break;
            const uint32_t idesc_h = (vm && (w.nu & 1) && h == mnh - 1) ? P.idesc128 : P.idesc;
            if (NH > 1 && kb == kb0) {      // column half h of the accumulator drained?
              const long long ch = trace ? clock64() : 0;
              mbar_wait(tempty0 + 8 * h, (it & 1) ^ 1);
              if (trace && pair_gid + u * nclusters * NPP < P.trace_n)
                trace[8 * (pair_gid + u * nclusters * NPP) + 5] += (unsigned long long)(clock64() - ch);
              tc_fence_after();
            }
#pragma unroll
            for (int k = 0; k < BK / 16; ++k) {
              const uint64_t ad = P.a_mn_major ? sdesc(a0 + 2048 * k, 8192, 1024) : sdesc(a0 + 32 * k, 16, 1024);
              const uint32_t bh = b0 + h * B2_BYTES;
              const uint64_t bd = P.b_mn_major ? sdesc(bh + 2048 * k, 8192, 1024) : sdesc(bh + 32 * k, 16, 1024);
              mma_bf16_cg2(d + 256 * h, ad, bd, idesc_h, (kb != kb0) || k != 0);
            }
          }
          if (CL == 4) mma_commit_cg2_mask(empty0 + 8 * stage, 0xF);
          else mma_commit_cg2(empty0 + 8 * stage);
          if (++stage == NS) { stage = 0; phase ^= 1; }
        }
        mma_commit_cg2_mask(tfull0 + 8 * acc, (uint16_t)(3u << (2 * pp)));
        if (trace && pair_gid + u * nclusters * NPP < P.trace_n) {
          trace[8 * (pair_gid + u * nclusters * NPP) + 2] = gtimer();
          // low word: cycles waiting for full stages; high word: cycles from the first wait to
          // the last MMA issued (the SM clock of this tile follows from mma_us)
          trace[8 * (pair_gid + u * nclusters * NPP) + 4] =
              (unsigned long long)(wfull & 0xffffffffll) | ((unsigned long long)(clock64() - cfirst) << 32);
        }
      }
      // drain: the last accumulators must be released before the barriers go away
      if (NH == 1) {
        for (int k = 0; k < 2 && it - 1 - k >= 0; ++k) {
          const int j = it - 1 - k;
          mbar_wait(tempty0 + 8 * (j & 1), (j >> 1) & 1);
        }
      } else if (it > 0) {
        mbar_wait(tempty0, (it - 1) & 1);
        mbar_wait(tempty0 + 8, (it - 1) & 1);
      }
    }
  } else {
    // ===== epilogue (both CTAs): this CTA's 128 accumulator rows =====
    const int quad = warp & 3;
    const int half = (warp - 2) >> 2;
    const int row = quad * 32 + lane;
    const int ew = rank * 8 + (warp - 2);          // this warp's slot in a stream-K partial
    // (1024-byte aligned: the TMA 128B swizzle pattern is a function of the address bits)
    const uint32_t stg0 = smem_u32(smem + NS * (A2_BYTES + BSTG) + 1024) + (warp - 2) * (EPB * 4096);
    int sbuf = 0;                                  // staging buffer of the next TMA store
    const uint32_t tempty_leader = map_to_rank(tempty0, 2 * pp);
    int it = 0;
    SkIter<LEAN> wi(P, cluster_id, nclusters);
    SkWork w;
    for (; wi.next(&w); ++it) {
      const int t = w.t;
      const int role = LEAN ? 0 : w.role;
      const int acc = NH == 1 ? it & 1 : 0;
      const int64_t m = vm ? (int64_t)t * 256 + rank * 128 + row
                                : ((int64_t)(t / P.tiles_n) * NPP + pp) * 256 + rank * 128 + row;
      const int64_t ntile = vm ? (int64_t)128 * w.u0 : (int64_t)(t % P.tiles_n) * NW;
      // columns of this tile held by this warp group in MMA half h (vmode: a group may hold none)
      auto group_has = [&](int h) { return !vm || 2 * h + half < w.nu; };
      mbar_wait(tfull0 + 8 * acc, NH == 1 ? (it >> 1) & 1 : it & 1);
      tc_fence_after();
      const bool mok = m < P.M;
      const int64_t crow = P.cbase + (OUT_ROWMAJOR ? (mok ? m : 0) * P.ldc : __ldg(P.cM + (mok ? m : 0)));
      // stream-K partials: warp ew of a pair's slot holds its 32 rows × 128 columns as
      // float4 [c][j][lane] (each store / load instruction covers 512 contiguous bytes)
      float4* mine = reinterpret_cast<float4*>(P.skpart + (int64_t)pair_gid * (NH * 65536) + ew * (NH * 4096)) + lane;
      int q1 = cluster_id;                           // finisher: partials of pairs cluster_id+1 .. q1
      if (role == 2) {
        const int64_t tend = (int64_t)(t - P.nfull + 1) * P.num_kb;
        while (q1 + 1 < P.sk_pairs && (int64_t)(q1 + 1) * P.sk_w / P.sk_pairs < tend) ++q1;
        if (lane == 0)
          for (int q = cluster_id + 1; q <= q1; ++q)
            while (*((volatile unsigned*)(P.skflag + (q * NPP + pp) * 16 + ew)) == 0u) __nanosleep(64);
        __syncwarp();
        __threadfence();
        if (trace && leader && warp == 2 && lane == 0 && pair_gid + it * nclusters * NPP < P.trace_n)
          trace[8 * (pair_gid + it * nclusters * NPP) + 6] = gtimer();
      }
      auto epi_chunk = [&](uint32_t* r, int64_t nb, int pc) {
        // fold the producers' partials in k order, two partials' loads in flight at a time
        // (the fold is latency-bound: 16 independent 512-byte warp loads per round trip)
        auto part = [&](int q) {
          return reinterpret_cast<const float4*>(P.skpart + (int64_t)(q * NPP + pp) * (NH * 65536) + ew * (NH * 4096)) +
                 lane + pc * 8 * 32;
        };
        int q = cluster_id + 1;
        for (; q + 1 <= q1; q += 2) {
          const float4* s0 = part(q);
          const float4* s1 = part(q + 1);
          float4 b0[8], b1[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) b0[j] = __ldcg(s0 + j * 32);
#pragma unroll
          for (int j = 0; j < 8; ++j) b1[j] = __ldcg(s1 + j * 32);
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            r[4 * j] = __float_as_uint(__uint_as_float(r[4 * j]) + b0[j].x + b1[j].x);
            r[4 * j + 1] = __float_as_uint(__uint_as_float(r[4 * j + 1]) + b0[j].y + b1[j].y);
            r[4 * j + 2] = __float_as_uint(__uint_as_float(r[4 * j + 2]) + b0[j].z + b1[j].z);
            r[4 * j + 3] = __float_as_uint(__uint_as_float(r[4 * j + 3]) + b0[j].w + b1[j].w);
          }
        }
        if (q <= q1) {
          const float4* s0 = part(q);
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const float4 b = __ldcg(s0 + j * 32);
            r[4 * j] = __float_as_uint(__uint_as_float(r[4 * j]) + b.x);
            r[4 * j + 1] = __float_as_uint(__uint_as_float(r[4 * j + 1]) + b.y);
            r[4 * j + 2] = __float_as_uint(__uint_as_float(r[4 * j + 2]) + b.z);
            r[4 * j + 3] = __float_as_uint(__uint_as_float(r[4 * j + 3]) + b.w);
          }
        }
        if (LEAN || (OUT_ROWMAJOR && P.c_vec4)) {   // (LEAN launches only with the TMA store map)
          // this warp's 32 rows × 32 columns into a 128B-swizzled staging image (16-byte chunk
          // j of row r at (j ^ (r & 7))·16: conflict-free), then one TMA tensor store of the
          // 32×32 box (rows / columns beyond M / N are clipped by the TMA unit); two staging
          // buffers per warp, so a buffer is rewritten only after its previous store read it
          const uint32_t stg = stg0 + sbuf * 4096;
          if (lane == 0) {
            if (EPB == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
            else asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
          }
          __syncwarp();
#pragma unroll
          for (int j = 0; j < 8; ++j)
            asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(stg + lane * 128 + ((j ^ (lane & 7)) << 4)),
                         "r"(r[4 * j]), "r"(r[4 * j + 1]), "r"(r[4 * j + 2]), "r"(r[4 * j + 3])
                         : "memory");
          fence_proxy_async();
          __syncwarp();
          if (lane == 0) {
            tma_store_2d(&mapC, stg, (int)nb, (int)(m - row + quad * 32));
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
          }
          sbuf ^= EPB - 1;
        } else if (OUT_ROWMAJOR && mok && nb + 32 <= P.N && ((crow + nb) & 3) == 0) {
          float4* dst = reinterpret_cast<float4*>(P.C + crow + nb);
#pragma unroll
          for (int j = 0; j < 8; ++j)
            dst[j] = make_float4(__uint_as_float(r[4 * j]), __uint_as_float(r[4 * j + 1]), __uint_as_float(r[4 * j + 2]),
                                 __uint_as_float(r[4 * j + 3]));
        } else if (mok) {
#pragma unroll
          for (int j = 0; j < 32; ++j)
            if (nb + j < P.N) P.C[crow + (OUT_ROWMAJOR ? nb + j : __ldg(P.cN + nb + j))] = __uint_as_float(r[j]);
        }
      };
#pragma unroll 1
      for (int h = 0; h < NH; ++h) {
      if (!group_has(h)) {             // nothing of this half for this group: release it at once
        if (NH > 1) {
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive_cluster(tempty_leader + 8 * h);
        }
        continue;
      }
      const int64_t n0 = ntile + 256 * h + half * 128;
      const uint32_t tb = tmem + ((uint32_t)(quad * 32) << 16) + acc * BN + 256 * h + half * 128;
      // (a software-pipelined variant — TMEM load of chunk c+1 in flight while chunk c is
      // stored — measured 1-3 % slower: the epilogue is bound by the memory system, not by
      // the TMEM load latency)
#pragma unroll 1
      for (int c = 0; c < 4; ++c) {
        uint32_t r[32];
        tmem_ld32(tb + c * 32, r);
        const int64_t nb = n0 + c * 32;
        const int pc = h * 4 + c;                    // 32-column chunk index in the partial
        if (role == 1) {
#pragma unroll
          for (int j = 0; j < 8; ++j)
            mine[(pc * 8 + j) * 32] = make_float4(__uint_as_float(r[4 * j]), __uint_as_float(r[4 * j + 1]),
                                                  __uint_as_float(r[4 * j + 2]), __uint_as_float(r[4 * j + 3]));
        } else {
          epi_chunk(r, nb, pc);
        }
      }
      if (NH > 1) {                    // column half h read out: the next tile may write it
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive_cluster(tempty_leader + 8 * h);
      }
      }
      if (role == 1) {               // publish this warp's part of the partial tile
        __threadfence();
        __syncwarp();
        if (lane == 0) atomicExch(P.skflag + pair_gid * 16 + ew, 1u);
        if (trace && leader && warp == 2 && lane == 0 && pair_gid + it * nclusters * NPP < P.trace_n)
          trace[8 * (pair_gid + it * nclusters * NPP) + 7] = gtimer();
      } else if (role == 2 && lane == 0) {
        for (int q = cluster_id + 1; q <= q1; ++q) P.skflag[(q * NPP + pp) * 16 + ew] = 0u;   // consumed: back to rest
      }
      if (NH == 1) {
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive_cluster(tempty_leader + 8 * acc);
      }
      if (trace && leader && warp == 2 && lane == 0 && pair_gid + it * nclusters * NPP < P.trace_n)
        trace[8 * (pair_gid + it * nclusters * NPP) + 3] = gtimer();
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");   // stores done before exit
  }
  __syncwarp();                  // lanes 1..31 of warps 0/1 wait for their role lane
  tc_fence_before();
  asm volatile("barrier.cluster.arrive.release;\n\tbarrier.cluster.wait.acquire;" ::: "memory");
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS));
  }
  if (trace && threadIdx.x == 0 && pair_gid < 256) trace[8 * P.trace_n + 2 * pair_gid + 1 + rank * 512] = gtimer();
}

// Few-tile split-K (1-SM kernel, P.xfold): S splits of each of the T tiles wrote dense
// fp32 partial tiles [128][256]; fold them in split order (deterministic) across the whole
// GPU and write through out_view (row-major or the offset tables; fp32 or bf16).
__global__ void __launch_bounds__(256) t4_xfold_kernel(const __grid_constant__ Params P) {
  asm volatile("griddepcontrol.wait;" ::: "memory");   // the GEMM grid's partials are visible
  constexpr int64_t PT = (int64_t)BM * BN;
  const int64_t per_tile = PT / 4;
  const int64_t total = (int64_t)(P.nunits / P.ssplit) * per_tile;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t ti = e / per_tile, q = e % per_tile;
    const int r = (int)(q / (BN / 4)), c4 = (int)(q % (BN / 4)) * 4;
    const float* src = P.part + ti * P.ssplit * PT + (int64_t)r * BN + c4;
    float4 a = __ldcg(reinterpret_cast<const float4*>(src));
    for (int sp = 1; sp < P.ssplit; ++sp) {
      const float4 b = __ldcg(reinterpret_cast<const float4*>(src + sp * PT));
      a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
    }
    int mb, nb;
    t_decode(P, P.nfull + (int)ti, &mb, &nb);
    const int64_t m = (int64_t)mb * BM + r;
    if (m >= P.M) continue;
    const int64_t row = P.cbase + (P.c_rowmajor ? m * P.ldc : P.cM[m]);
    const float v[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int64_t n = (int64_t)nb * BN + c4 + j;
      if (n >= P.N) break;
      const int64_t o = row + (P.c_rowmajor ? n : P.cN[n]);
      if (P.out_bf16) ((__nv_bfloat16*)P.C)[o] = __float2bfloat16_rn(v[j]);
      else P.C[o] = v[j];
    }
  }
}

constexpr int SK_MAX_PAIRS = 74;     // stream-K partial slots reserved in the workspace (2-SM path)
constexpr int SK_MIN_SEG = 8;        // shortest stream-K range per pair, in 64-deep k-blocks
constexpr int MAX_TAIL_UNITS1 = 296; // 1-SM path: bound on tail units (partials sized per plan)

// ---- operand normalisation pre-pass ---------------------------------------------------
// An operand whose (MN, K) offsets are not 2-D linear (e.g. CCSD(T)'s t2 in output order,
// the stride-2 im2col view of an MCC image) is gathered once per execute into a 2-D
// K-major [MN][ld] (or MN-major [K][ld]) bf16 copy in the workspace; the GEMM then reads
// it with TMA.  16-byte chunks when the source is contiguous along the inner dim.
struct PermParams {
  const uint16_t* src;
  uint16_t* dst;
  const int64_t* offO;   // outer-dim offsets (MN for K-major, K for MN-major)
  const int64_t* offI;   // inner-dim offsets
  int64_t nO, nI, ld;
  int chunked;           // inner offsets contiguous in runs of 8 (aligned)
};

// chunked gather with a 2-D grid (blockIdx.y = outer row): no integer division per chunk,
// two independent 16-byte chunks per thread in flight
__global__ void __launch_bounds__(256) permute_rows_kernel(const __grid_constant__ PermParams P) {
  const int64_t o = blockIdx.y;
  const int64_t nc = P.nI / 8;
  const uint16_t* src = P.src + P.offO[o];
  uint16_t* dst = P.dst + o * P.ld;
  const int64_t span = 2 * (int64_t)blockDim.x;
  for (int64_t c = (int64_t)blockIdx.x * span + threadIdx.x; c < nc; c += (int64_t)gridDim.x * span) {
    const int64_t c2 = c + blockDim.x;
    const uint4 v0 = __ldg(reinterpret_cast<const uint4*>(src + __ldg(P.offI + c * 8)));
    uint4 v1 = v0;
    if (c2 < nc) v1 = __ldg(reinterpret_cast<const uint4*>(src + __ldg(P.offI + c2 * 8)));
    *reinterpret_cast<uint4*>(dst + c * 8) = v0;
    if (c2 < nc) *reinterpret_cast<uint4*>(dst + c2 * 8) = v1;
  }
}

// chunked gather, one warp per outer row: 32-bit chunk indices, 4 independent 16-byte loads
// in flight per lane, coalesced stores along the row
__global__ void __launch_bounds__(256) permute_warp_kernel(const __grid_constant__ PermParams P) {
  const int lane = threadIdx.x & 31;
  const int nc = (int)(P.nI / 8);
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t o = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); o < P.nO; o += warps) {
    const uint16_t* src = P.src + P.offO[o];
    uint16_t* dst = P.dst + o * P.ld;
    int c = lane;
    for (; c + 96 < nc; c += 128) {
      uint4 v[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) v[u] = __ldg(reinterpret_cast<const uint4*>(src + __ldg(P.offI + (int64_t)(c + 32 * u) * 8)));
#pragma unroll
      for (int u = 0; u < 4; ++u) *reinterpret_cast<uint4*>(dst + (int64_t)(c + 32 * u) * 8) = v[u];
    }
    for (; c < nc; c += 32)
      *reinterpret_cast<uint4*>(dst + (int64_t)c * 8) = __ldg(reinterpret_cast<const uint4*>(src + __ldg(P.offI + (int64_t)c * 8)));
  }
}

__global__ void __launch_bounds__(256) permute_kernel(const __grid_constant__ PermParams P) {
  if (P.chunked) {
    const int64_t nc = P.nI / 8;
    const int64_t total = P.nO * nc;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
      const int64_t o = e / nc, c = e % nc;
      const uint4 v = __ldg(reinterpret_cast<const uint4*>(P.src + P.offO[o] + P.offI[c * 8]));
      *reinterpret_cast<uint4*>(P.dst + o * P.ld + c * 8) = v;
    }
  } else {
    const int64_t total = P.nO * P.nI;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
      const int64_t o = e / P.nI, i = e % P.nI;
      P.dst[o * P.ld + i] = P.src[P.offO[o] + __ldg(P.offI + i)];
    }
  }
}

// ------------------------------------------------------------------------- host
struct Layout2D {
  bool ok = false;
  bool mn_major = false;       // unit stride along M (N) instead of K
  int64_t ld = 0;              // stride (elements) of the non-unit dim
  bool permuted = false;       // gathered into the workspace by permute_kernel
  int chunked = 0;
  size_t ws_off = 0;
};

static bool linear(const std::vector<int64_t>& t, int64_t* stride) {
  if (t.size() <= 1) { *stride = 0; return true; }
  int64_t s = t[1] - t[0];
  for (size_t i = 1; i < t.size(); ++i)
    if (t[i] - t[i - 1] != s) return false;
  *stride = s;
  return true;
}

static std::vector<int64_t> table(const Plan& p, const int* dims, int nd, const Access& acc) {
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

static Layout2D operand_layout(const Plan& p, const int* mdims, int nmd, int64_t MN, const Access& acc, std::string* why,
                               const char* name) {
  Layout2D L;
  int64_t smn, sk;
  const Contraction& c = p.con;
  if (!linear(table(p, mdims, nmd, acc), &smn) || !linear(table(p, c.kd, c.nk, acc), &sk)) {
    *why = std::string(name) + " offsets are not 2-D linear";
    return L;
  }
  if (MN == 1) smn = 1;
  if (c.K == 1) sk = 1;
  if (sk == 1 && (smn * 2) % 16 == 0 && smn > 0) { L.ok = true; L.mn_major = false; L.ld = smn; }
  else if (smn == 1 && (sk * 2) % 16 == 0 && sk > 0) { L.ok = true; L.mn_major = true; L.ld = sk; }
  else *why = std::string(name) + " has no unit stride with a 16-byte aligned leading dimension (TMA)";
  return L;
}

}  // namespace t4

// direct TMA operand, or a planned gather into a 2-D layout (operand normalisation)
static t4::Layout2D plan_operand(const Plan& p, const int* mdims, int nmd, int64_t MN, const Access& acc,
                                 std::string* why, const char* name, size_t* ws) {
  t4::Layout2D L = t4::operand_layout(p, mdims, nmd, MN, acc, why, name);
  if (L.ok && acc.base % 8 == 0) return L;
  const Contraction& c = p.con;
  std::vector<int64_t> tk = t4::table(p, c.kd, c.nk, acc), tm = t4::table(p, mdims, nmd, acc);
  auto runs8 = [&](const std::vector<int64_t>& t) {
    if (t.size() % 8) return false;
    for (size_t i = 0; i < t.size(); i += 8) {
      if ((t[i] + acc.base) % 8) return false;
      for (int j = 1; j < 8; ++j)
        if (t[i + j] != t[i] + j) return false;
    }
    return true;
  };
  L = t4::Layout2D();
  L.ok = true;
  L.permuted = true;
  if (runs8(tk) || !runs8(tm)) {        // K-major copy [MN][ld]
    L.mn_major = false;
    L.ld = (c.K + 7) / 8 * 8;
    L.chunked = runs8(tk);
    *ws = (*ws + 255) / 256 * 256;
    L.ws_off = *ws;
    *ws += (size_t)MN * L.ld * 2;
  } else {                              // MN-major copy [K][ld]
    L.mn_major = true;
    L.ld = (MN + 7) / 8 * 8;
    L.chunked = 1;
    *ws = (*ws + 255) / 256 * 256;
    L.ws_off = *ws;
    *ws += (size_t)c.K * L.ld * 2;
  }
  return L;
}

bool t4_supported(const Plan& p, std::string* why) {
  const Contraction& c = p.con;
  if (c.Z != 1) { *why = "batched contraction (Z>1) not in the tcgen05 template yet"; return false; }
  if (p.out[0].dtype != MDH_F32 && p.out[0].dtype != MDH_BF16) { *why = "output must be f32/bf16"; return false; }
  if (c.M > INT32_MAX || c.N > INT32_MAX || c.K > INT32_MAX) { *why = "extent exceeds TMA coordinates"; return false; }
  size_t ws = 0;
  std::string w;
  t4::Layout2D a = plan_operand(p, c.md, c.nm, c.M, p.in[c.a_buf].acc[0], &w, "A", &ws);
  t4::Layout2D b = plan_operand(p, c.nd, c.nn, c.N, p.in[c.b_buf].acc[0], &w, "B", &ws);
  *why = std::string("A ") + (a.permuted ? "gathered " : "") + (a.mn_major ? "MN" : "K") + "-major, B " +
         (b.permuted ? "gathered " : "") + (b.mn_major ? "MN" : "K") + "-major";
  return true;
}

struct T4State {
  t4::Layout2D a, b;
  t4::Params P;
  int cg = 1;      // 1: one SM per 128×256 tile; 2: SM pair per 256×256 tile
  int cl = 2;      // 2-SM kernel: CTAs per cluster (4: two pairs share B by multicast)
  int nw = 256;    // 2-SM kernel: N extent of a pair tile (512: two MMAs per k-step)
  int wst = 4;     // wide 2-SM ring stages (4: single-buffered epilogue staging; tile knob stages=3: double-buffered)
  bool sk_ok = false;   // 2-SM kernel: stream-K workspace reserved
  bool ag = false; // A staged by the kernel's gather warps (no A tensor map, no pre-pass)
  bool ic = false;  // A through a TMA im2col map
  uint64_t ic_dims[4];
  int ic_upper[2];
  uint32_t ic_estr[4];
  int epi = 1;      // 0 row-major C, 1 per-element scatter, 2 run-8 vector scatter, 3 bulk runs
  size_t smem3 = 0; // dynamic shared memory of the EPI 3 kernel
  int tail_parts = 0;   // 1-SM split-K tail: partial tiles in the workspace at tail_off
  int grid1 = 0;        // its grid (the SM count at plan time: one tail unit per CTA)
  size_t tail_off = 0;
  // implicit-GEMM A map (a_box): TMA-order dims, byte strides, box
  int brank = 0;
  uint64_t bdims[5], bstrides[4];
  uint32_t bbox[5];
};

static int plan_sms(const Plan* p) {
  int sms = 148;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, p->device) != cudaSuccess || sms <= 0) {
    cudaGetLastError();
    sms = 148;
  }
  return sms;
}

// Implicit-GEMM planning for A (e.g. MCC's img[n, 2p+r, 2q+s, c]): pick g* (an M dim with a
// unit coefficient on one buffer coordinate, extent a multiple of the 128-row tile) and k*
// (a K dim with a unit coefficient on the innermost buffer coordinate, extent a multiple of
// the 64-deep k-block); reorder the M and K groups so g* and k* are innermost.  Returns
// false (operand then gathered or 2-D) when the index function has no such pair.
static bool plan_box(Plan* p, T4State* s) {
  Contraction& c = p->con;
  const Buf& Ab = p->in[c.a_buf];
  const mdh_index_fn& fn = Ab.fn[0];
  const int R = Ab.rank;
  if (R < 3 || R > 5 || Ab.dtype != MDH_BF16 || (Ab.shape[R - 1] * 2) % 16) return false;
  auto unit_coord = [&](int d) {
    int r0 = -1;
    for (int r = 0; r < R; ++r)
      if (fn.coeff[r][d] != 0) {
        if (r0 >= 0 || fn.coeff[r][d] != 1) return -2;
        r0 = r;
      }
    return r0;
  };
  int g = -1, gi = -1, k = -1, ki = -1, rg = -1;
  for (int i = 0; i < c.nm; ++i) {
    const int d = c.md[i], r = unit_coord(d);
    if (r >= 0 && p->size[d] % 128 == 0 && (g < 0 || p->size[d] > p->size[g])) { g = d; gi = i; rg = r; }
  }
  for (int i = 0; i < c.nk; ++i) {
    const int d = c.kd[i], r = unit_coord(d);
    if (r == R - 1 && p->size[d] % 64 == 0) { k = d; ki = i; }
  }
  if (g < 0 || k < 0 || rg == R - 1 || c.nm - 1 > 4 || c.nk - 1 > 4) return false;
  // reorder: g* innermost in M, k* innermost in K (B's K order follows, checked afterwards)
  for (int i = gi; i < c.nm - 1; ++i) c.md[i] = c.md[i + 1];
  c.md[c.nm - 1] = g;
  for (int i = ki; i < c.nk - 1; ++i) c.kd[i] = c.kd[i + 1];
  c.kd[c.nk - 1] = k;
  t4::BoxGen& B = s->P.abox;
  memset(&B, 0, sizeof(B));
  B.rank = R;
  B.jg = R - 1 - rg;
  B.jk = 0;
  B.gsize = p->size[g];
  B.ksize = p->size[k];
  B.ng = c.nm - 1;
  B.nk = c.nk - 1;
  for (int o = 0; o < B.ng; ++o) {
    B.gdim[o] = p->size[c.md[o]];
    for (int j = 0; j < R; ++j) B.gco[o][j] = (int)fn.coeff[R - 1 - j][c.md[o]];
  }
  for (int q = 0; q < B.nk; ++q) {
    B.kdim[q] = p->size[c.kd[q]];
    for (int j = 0; j < R; ++j) B.kco[q][j] = (int)fn.coeff[R - 1 - j][c.kd[q]];
  }
  for (int j = 0; j < R; ++j) B.base[j] = (int)fn.offset[R - 1 - j];
  s->brank = R;
  int64_t stride = 2;
  for (int j = 0; j < R; ++j) {
    s->bdims[j] = (uint64_t)Ab.shape[R - 1 - j];
    if (j > 0) s->bstrides[j - 1] = (uint64_t)stride;
    stride *= Ab.shape[R - 1 - j];
    s->bbox[j] = j == B.jk ? 64u : (j == B.jg ? 128u : 1u);
  }
  return true;
}

// TMA im2col planning for A (MCC's img[n, σh·p + r, σw·q + s, c], Listing 12): rank-4 NHWC
// bf16 buffer, M group (n,) p, q and K group r, s, c in that order, C % 64 == 0.
static bool plan_im2col(const Plan* p, T4State* s) {
  const Contraction& c = p->con;
  const Buf& Ab = p->in[c.a_buf];
  if (Ab.rank != 4 || Ab.dtype != MDH_BF16 || c.nk != 3 || (c.nm != 2 && c.nm != 3)) return false;
  const mdh_index_fn& fn = Ab.fn[0];
  const int dn = c.nm == 3 ? c.md[0] : -1, dp = c.md[c.nm - 2], dq = c.md[c.nm - 1];
  const int dr = c.kd[0], ds = c.kd[1], dc = c.kd[2];
  int64_t want[4][MDH_MAX_D] = {};
  if (dn >= 0) want[0][dn] = 1;
  want[1][dp] = fn.coeff[1][dp];
  want[1][dr] = 1;
  want[2][dq] = fn.coeff[2][dq];
  want[2][ds] = 1;
  want[3][dc] = 1;
  for (int r = 0; r < 4; ++r) {
    if (fn.offset[r] != 0) return false;
    for (int d = 0; d < p->D; ++d)
      if (p->size[d] > 1 && fn.coeff[r][d] != want[r][d]) return false;
  }
  const int64_t sh = fn.coeff[1][dp], sw = fn.coeff[2][dq];
  const int64_t C = Ab.shape[3], H = Ab.shape[1], W = Ab.shape[2];
  if (sh < 1 || sh > 8 || sw < 1 || sw > 8 || p->size[dc] != C || C % 64) return false;
  const int64_t P = p->size[dp], Q = p->size[dq], S = p->size[ds];
  const int64_t uh = sh * (P - 1) - (H - 1), uw = sw * (Q - 1) - (W - 1);
  if (uh < -128 || uh > 127 || uw < -128 || uw > 127) return false;
  s->ic_dims[0] = (uint64_t)C;
  s->ic_dims[1] = (uint64_t)W;
  s->ic_dims[2] = (uint64_t)H;
  s->ic_dims[3] = (uint64_t)Ab.shape[0];
  s->ic_upper[0] = (int)uw;
  s->ic_upper[1] = (int)uh;
  s->ic_estr[0] = 1;
  s->ic_estr[1] = (uint32_t)sw;
  s->ic_estr[2] = (uint32_t)sh;
  s->ic_estr[3] = 1;
  t4::Params& Pp = s->P;
  Pp.a_im2col = 1;
  Pp.ic_C = (int)C;
  Pp.ic_P = (int)P;
  Pp.ic_Q = (int)Q;
  Pp.ic_S = (int)S;
  Pp.ic_sh = (int)sh;
  Pp.ic_sw = (int)sw;
  return true;
}

mdh_status prepare_t4(Plan* p) {
  std::string why;
  if (!t4_supported(*p, &why)) { set_error("T4: %s", why.c_str()); return MDH_ERR_UNSUPPORTED; }
  if (prepare_t4_conv(p)) return MDH_OK;           // small-K direct variant (t4_conv.cu)
  const Contraction& c = p->con;
  T4State* s = new T4State();
  s->wst = p->tiles.stages == 3 ? 3 : 4;
  size_t ws = 0;
  std::string w2;
  const t4::Layout2D a_direct = t4::operand_layout(*p, c.md, c.nm, c.M, p->in[c.a_buf].acc[0], &w2, "A");
  // implicit GEMM is opt-in (tile knob implicit=1): measured slower than the gather
  // pre-pass on MCC conv5_1
  const bool a_2d = a_direct.ok && p->in[c.a_buf].acc[0].base % 8 == 0;
  const bool a_box = !a_2d && p->tiles.implicit == 1 && plan_box(p, s);
  const t4::BoxGen box = s->P.abox;
  // TMA im2col (implicit 0 = auto or 4): the convolution operand straight from the image
  t4::Params icp;
  memset(&icp, 0, sizeof(icp));
  s->P = icp;
  const bool a_ic = !a_2d && !a_box && (p->tiles.implicit == 0 || p->tiles.implicit == 4) && plan_im2col(p, s);
  icp = s->P;
  s->ic = a_ic;
  // in-kernel gather (implicit 0 = auto or 2): A's K offsets in aligned runs of 8, so each
  // 16-byte chunk of a swizzled A row is one cp.async
  bool a_gather = false;
  if (!a_2d && !a_box && !a_ic && (p->tiles.implicit == 0 || p->tiles.implicit == 2) && c.K % 8 == 0 &&
      c.K / 8 <= t4::KOFF_MAX) {
    std::vector<int64_t> tk = t4::table(*p, c.kd, c.nk, p->in[c.a_buf].acc[0]);
    std::vector<int64_t> tm = t4::table(*p, c.md, c.nm, p->in[c.a_buf].acc[0]);
    const int64_t base = p->in[c.a_buf].acc[0].base;
    a_gather = true;
    for (size_t i = 0; i < tk.size() && a_gather; i += 8) {
      if ((tk[i] + base) % 8) a_gather = false;
      for (int j = 1; j < 8 && a_gather; ++j)
        if (tk[i + j] != tk[i] + j) a_gather = false;
    }
    for (size_t i = 0; i < tm.size() && a_gather; ++i)
      if (tm[i] % 8) a_gather = false;
  }
  // 8-byte gather: K offsets contiguous only in aligned runs of 4 (MCC_Caps' capsule dim l)
  bool a_gather4 = false;
  if (!a_2d && !a_box && !a_ic && !a_gather && (p->tiles.implicit == 0 || p->tiles.implicit == 2) && c.K % 4 == 0 &&
      c.K / 4 <= t4::KOFF_MAX) {
    std::vector<int64_t> tk = t4::table(*p, c.kd, c.nk, p->in[c.a_buf].acc[0]);
    std::vector<int64_t> tm = t4::table(*p, c.md, c.nm, p->in[c.a_buf].acc[0]);
    const int64_t base = p->in[c.a_buf].acc[0].base;
    a_gather4 = true;
    for (size_t i = 0; i < tk.size() && a_gather4; i += 4) {
      if ((tk[i] + base) % 4) a_gather4 = false;
      for (int j = 1; j < 4 && a_gather4; ++j)
        if (tk[i + j] != tk[i] + j) a_gather4 = false;
    }
    for (size_t i = 0; i < tm.size() && a_gather4; ++i)
      if (tm[i] % 4) a_gather4 = false;
    if (a_gather4) a_gather = true;
  }
  if (a_box || a_gather || a_ic) {
    s->a = t4::Layout2D();
    s->a.ok = true;
  } else {
    s->a = plan_operand(*p, c.md, c.nm, c.M, p->in[c.a_buf].acc[0], &why, "A", &ws);
  }
  s->b = plan_operand(*p, c.nd, c.nn, c.N, p->in[c.b_buf].acc[0], &why, "B", &ws);
  int64_t akc, bkc;
  p->host_const.clear();
  build_contraction_tables(p, &akc, &bkc);
  t4::Params& P = s->P;
  memset(&P, 0, sizeof(P));
  P.a_box = a_box;
  P.abox = box;
  // (off by default: on MCC conv5_1 it measured 89 vs 98 µs on one box and 103 vs 88.5 on
  // another; MatMul 4096³ 1048 vs 1266 TFLOP/s)
  P.krot = p->tiles.krot > 0 ? 1 : 0;
  P.a_im2col = icp.a_im2col;
  P.ic_C = icp.ic_C;
  P.ic_P = icp.ic_P;
  P.ic_Q = icp.ic_Q;
  P.ic_S = icp.ic_S;
  P.ic_sh = icp.ic_sh;
  P.ic_sw = icp.ic_sw;
  P.M = c.M;
  P.N = c.N;
  P.K = c.K;
  P.tiles_m = (int)((c.M + t4::BM - 1) / t4::BM);
  P.tiles_n = (int)((c.N + t4::BN - 1) / t4::BN);
  P.num_tiles = P.tiles_m * P.tiles_n;
  P.num_kb = (int)((c.K + t4::BK - 1) / t4::BK);
  P.a_mn_major = s->a.mn_major;
  P.b_mn_major = s->b.mn_major;
  // instruction descriptor (kind::f16): D f32, A/B bf16, majors, N>>3, M>>4
  P.idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)P.a_mn_major << 15) | ((uint32_t)P.b_mn_major << 16) |
            ((uint32_t)(t4::BN >> 3) << 17) | ((uint32_t)(t4::BM >> 4) << 24);
  P.out_bf16 = p->out[0].dtype == MDH_BF16;
  // is C row-major over (m, n)?  cM[m] = m*ldc, cN[n] = n
  std::vector<int64_t> cm = t4::table(*p, c.md, c.nm, p->out[0].acc[0]);
  std::vector<int64_t> cn = t4::table(*p, c.nd, c.nn, p->out[0].acc[0]);
  int64_t sm = 0, sn = 0;
  bool lm = t4::linear(cm, &sm), ln = t4::linear(cn, &sn);
  if (c.N == 1) sn = 1;
  P.c_rowmajor = lm && ln && sn == 1 && cm[0] == 0 && cn[0] == 0;
  P.ldc = sm;
  P.cbase = p->out[0].acc[0].base;
  P.sched = P.c_rowmajor ? 0 : 1;
  // run-8 scatter epilogue (EPI 2): cN in aligned runs of 8 consecutive elements and every
  // row offset a multiple of 8, so a thread's 8 consecutive accumulators are one vector
  s->epi = P.c_rowmajor ? 0 : 1;
  if (!P.c_rowmajor && c.N % 8 == 0) {
    bool run8 = true;
    for (size_t i = 0; i < cn.size() && run8; i += 8) {
      if ((P.cbase + cn[i]) % 8) run8 = false;
      for (int j = 1; j < 8 && run8; ++j)
        if (cn[i + j] != cn[i] + j) run8 = false;
    }
    for (size_t i = 0; i < cm.size() && run8; ++i)
      if (cm[i] % 8) run8 = false;
    if (run8) s->epi = 2;
  }
  // run-4 variant (fp32 output; MCC_Caps: res[…, k, i, j] with j the 4-run between k and i)
  if (!P.c_rowmajor && s->epi == 1 && c.N % 4 == 0 && p->out[0].dtype == MDH_F32) {
    bool run4 = true;
    for (size_t i = 0; i < cn.size() && run4; i += 4) {
      if ((P.cbase + cn[i]) % 4) run4 = false;
      for (int j = 1; j < 4 && run4; ++j)
        if (cn[i + j] != cn[i] + j) run4 = false;
    }
    for (size_t i = 0; i < cm.size() && run4; ++i)
      if (cm[i] % 4) run4 = false;
    if (run4) {
      s->epi = 2;
      P.run4 = 1;
    }
  }
  // 2-SM pairs (cta_group::2, 256×256 tiles) for large row-major outputs (measured 1290 vs
  // 1170 TFLOP/s on MatMul 4096³); tile knob cluster=1 forces the 1-SM kernel
  // (the in-kernel A gather is a 1-SM kernel: a 2-SM version, whose peer CTA must publish
  // its gathered half at cluster scope, measured 86-208 µs vs 83 µs on MCC conv5_1)
  s->ag = a_gather;
  P.ag4 = a_gather4 ? 1 : 0;
  P.nkc = (int)(c.K / (a_gather4 ? 4 : 8));
  s->cg = (!a_gather && P.c_rowmajor && !P.out_bf16 && c.M >= 256 && c.N >= 256 && p->tiles.cluster != 1) ? 2 : 1;
  if (s->cg == 2) {
    P.tiles_m = (int)((c.M + 255) / 256);
    P.tiles_n = (int)((c.N + 255) / 256);
    P.num_tiles = P.tiles_m * P.tiles_n;
    P.idesc = (P.idesc & ~(0x1Fu << 24)) | ((uint32_t)(256 >> 4) << 24);
    // 4-CTA clusters (two pairs on a 512×256 super-tile sharing B; cuBLAS's 4096³ kernel is
    // 2cta with a 2×2 cluster): L2→SM operand traffic per k-block 24 instead of 32 KB per
    // CTA.  Opt-in (tile knob cluster=4): only 33 four-CTA clusters are co-resident on a
    // B200 (132 SMs), and the ~4 % faster k-block rate measured does not pay for the 16 idle
    // SMs (MatMul 4096³ 120.8 vs 110.7 µs, MCC conv5_1 74.5 vs 68.4 µs).
    if (P.tiles_m >= 2 && p->tiles.cluster == 4) {
      s->cl = 4;
      P.num_tiles = ((P.tiles_m + 1) / 2) * P.tiles_n;
    } else if (c.N > 256 && p->tiles.bn != 256 &&
               (p->tiles.bn == 512 || icp.a_im2col ||
                (int64_t)P.tiles_m * ((c.N + 511) / 512) >= std::max(1, plan_sms(p) / 2))) {
      // wide pair tiles 256×512: A is requested once per 8.4 MFLOP instead of
      // per 4.2.  Auto for an im2col A (MCC conv5_1) and for GEMMs with at least one full
      // wave of wide tiles (tools/sweep_tiles.py, whole tiles: 4096³ 106.6 vs 116.7 µs, 8192³
      // 717.7 vs 840.7 µs; 2048³, 32 wide tiles: narrow 24.6 vs 35.7 µs); tile knob bn=256|512
      s->nw = 512;
      P.tiles_n = (int)((c.N + 511) / 512);
      P.num_tiles = P.tiles_m * P.tiles_n;
    }
    // room for the stream-K partial tiles and flags, only when stream-K can be chosen at
    // launch (forced, or the auto rule: one partial wave of deep tiles — fewer tiles than
    // pairs, and the launch never has more pairs than SMs/2)
    s->sk_ok = p->tiles.split >= 2 || (p->tiles.split == 0 && P.num_tiles < plan_sms(p) / 2 && P.num_kb >= 64);
    if (s->sk_ok) {
      ws = (ws + 255) / 256 * 256;
      s->tail_off = ws;
      ws += (size_t)t4::SK_MAX_PAIRS * (s->nw / 256) * 65536 * sizeof(float) + 16 * t4::SK_MAX_PAIRS * sizeof(unsigned) + 256;
    }
  } else {
    // 1-SM split-K tail: the T mod C tiles of the last, partial wave split along K over
    // the idle SMs (S units each) — tile knob split=S, or automatically when the partial
    // wave is a large share of a K-deep contraction (MCC conv5_1: 196 tiles on 148 SMs)
    int dev = p->device, sms = 148;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms <= 0) {
      cudaGetLastError();
      sms = 148;
    }
    const int T = P.num_tiles, C = std::max(1, std::min(T, sms)), R = T / C, Tr = T - R * C;
    int S = 1;
    if (4 * T <= sms && P.num_kb >= 16 && p->tiles.split != 1) {
      // few tiles, deep K (MCC conv5_1 at the paper's N = 1: 2 tiles × 72 k-blocks): split
      // every tile along K over the idle SMs, all splits write partials, and a separate
      // grid-wide fold (t4_xfold_kernel) adds them in split order
      // (auto: at least 4 k-blocks per split; a forced split=S may go down to one)
      S = std::min({sms / T, p->tiles.split > 1 ? P.num_kb : P.num_kb / 4, t4::MAX_TAIL_UNITS1 / T});
      if (p->tiles.split > 1) S = std::min(S, p->tiles.split);
      if (S >= 2) {
        P.xfold = 1;
        P.sched = 0;
        P.nfull = 0;
        P.ssplit = S;
        P.nunits = T * S;
        ws = (ws + 255) / 256 * 256;
        s->tail_off = ws;
        ws += (size_t)T * S * t4::BM * t4::BN * sizeof(float) + 2 * (size_t)T * sizeof(unsigned) + 256;
        s->tail_parts = T * S;
        s->grid1 = std::min(T * S, sms);
        S = 1;                                   // (the tail logic below is skipped)
      }
    } else if (Tr > 0) {
      const int cap = std::min({C / Tr, P.num_kb / 4, t4::MAX_TAIL_UNITS1 / Tr});
      if (p->tiles.split > 1) S = std::min(p->tiles.split, cap);
      // (no automatic split: on MCC conv5_1 split 2/3/4 measured 84/92/92 µs vs 84 whole)
    }
    if (S >= 2) {
      P.sched = 0;
      P.nfull = T - Tr;
      P.ssplit = S;
      P.nunits = P.nfull + Tr * S;
      ws = (ws + 255) / 256 * 256;
      s->tail_off = ws;
      ws += (size_t)Tr * S * t4::BM * t4::BN * sizeof(float) + 2 * (size_t)Tr * sizeof(unsigned) + 256;
      s->tail_parts = Tr * S;
      s->grid1 = C;
    }
  }
  // bulk-run epilogue (EPI 3): the output is contiguous along n in runs of L elements
  // (cN[iL + j] = cN[iL] + j), 32 ≤ L ≤ 128, L % 8 == 0, N % L == 0, 16-byte aligned run
  // starts and row offsets; the N-tile becomes 2L wide so every tile holds whole runs and
  // a warp's rows go out as contiguous cp.async.bulk stores (CCSD(T): L = 72, bn = 144).
  // fp32 output, 1-SM kernel, TMA-fed A, K-major B, no split tail; tile knob epi=0 disables.
  P.bn = t4::BN;
  P.nstg = 0;
  P.e3flip = p->tiles.epi != 2;
  if (s->epi != 0 && !P.out_bf16 && s->cg == 1 && !a_gather && !a_box && !a_ic && !s->b.mn_major && s->tail_parts == 0 &&
      p->tiles.epi != 1) {
    int64_t L = 1;
    while (L < c.N && cn[(size_t)L] == cn[0] + L) ++L;
    bool ok = L >= 32 && L <= t4::EPI3_LMAX && L % 8 == 0 && c.N % L == 0;
    for (int64_t i = 0; i < c.N && ok; i += L) {
      if ((P.cbase + cn[(size_t)i]) % 4) ok = false;
      for (int64_t j = 1; j < L && ok; ++j)
        if (cn[(size_t)(i + j)] != cn[(size_t)i] + j) ok = false;
    }
    for (size_t i = 0; i < cm.size() && ok; ++i)
      if (cm[i] % 4) ok = false;
    if (ok) {
      const int bn = (int)(2 * L);
      const size_t stg1 = (size_t)8 * 32 * L * 4;
      const size_t lim = t4::SMEM_LIMIT - 1024 - t4::BN * sizeof(int64_t);
      // B resident when its whole K extent fits beside two A stages and double-buffered staging
      const size_t ring_res = 2 * (size_t)t4::A_BYTES + (size_t)P.num_kb * bn * 128;
      P.bres = p->tiles.epi != 3 && ring_res + 1024 + 2 * stg1 <= lim;
      const size_t ring = P.bres ? ring_res : 2 * ((size_t)t4::A_BYTES + (size_t)bn * 128);
      P.nstg = ring + 1024 + 2 * stg1 <= lim ? 2 : (ring + 1024 + stg1 <= lim ? 1 : 0);
      if (P.nstg > 0) {
        s->epi = 3;
        P.bn = bn;
        P.tiles_n = (int)((c.N + bn - 1) / bn);
        P.num_tiles = P.tiles_m * P.tiles_n;
        P.idesc = (P.idesc & ~(0x3Fu << 17)) | ((uint32_t)(bn >> 3) << 17);
        s->smem3 = ring + 1024 + P.nstg * stg1 + 1024;
      }
    }
  }
  if (s->epi == 3) P.krot = 0;      // the resident-B slots are indexed by the k-block itself
  p->tmaps = s;
  p->t4_variant = 1 + (s->a.permuted ? 2 : 0) + (s->b.permuted ? 4 : 0) + (s->cg == 2 ? 8 : 0) + (a_box ? 16 : 0) +
                  (a_gather ? 32 : 0) + (s->epi == 2 ? 64 : 0) + (s->epi == 3 ? 128 : 0) + (a_ic ? 256 : 0);
  p->ws_kernel = ws;
  p->tiles.bm = s->cg == 2 ? 256 : t4::BM;
  p->tiles.bn = s->epi == 3 ? P.bn : (s->cg == 2 ? s->nw : t4::BN);
  p->tiles.bk = t4::BK;
  p->tiles.stages = s->cg == 2 ? (s->nw == 512 ? s->wst : t4::S2) : (s->epi == 3 ? 2 : t4::STAGES);
  p->tiles.cluster = s->cg == 2 ? s->cl : 1;
  return MDH_OK;
}

void release_t4(Plan* p) {
  if (p->tmaps) {
    delete (T4State*)p->tmaps;
    p->tmaps = nullptr;
  }
}

static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeTiled_v12000)f;
  });
  return fn;
}

typedef CUresult (*EncodeIm2colFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const int*, const int*, cuuint32_t, cuuint32_t, const cuuint32_t*,
                                   CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                                   CUtensorMapFloatOOBfill);
static EncodeIm2colFn encode_im2col_fn() {
  static EncodeIm2colFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (EncodeIm2colFn)f;
  });
  return fn;
}

// im2col map of an NHWC bf16 image: 64 channels × 128 output pixels per load (SWIZZLE_128B
// rows, the K-major A tile layout); lower corner 0, upper corner so that the traversal
// visits exactly P (Q) window origins with strides (σh, σw)
static mdh_status make_im2col_map(CUtensorMap* map, const void* base, const T4State& s) {
  auto fn = encode_im2col_fn();
  if (!fn) { set_error("cuTensorMapEncodeIm2col unavailable"); return MDH_ERR_CUDA; }
  cuuint64_t strides[3] = {s.ic_dims[0] * 2, s.ic_dims[0] * s.ic_dims[1] * 2, s.ic_dims[0] * s.ic_dims[1] * s.ic_dims[2] * 2};
  int lower[2] = {0, 0};
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(base), s.ic_dims, strides, lower, s.ic_upper,
                  64, 128, s.ic_estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { set_error("cuTensorMapEncodeIm2col failed (%d)", (int)r); return MDH_ERR_CUDA; }
  return MDH_OK;
}

// diagnostics (MDH_T4_TRACE=1): a device buffer for the per-unit timeline of the last
// 2-SM launch, read back by mdh_debug_t4_trace
static unsigned long long* g_trace = nullptr;
static int g_trace_units = 0;
static int g_trace_used = 0;     // trace_n of the last traced launch (its entry/exit block follows)
static unsigned long long* t4_trace_buffer(int units) {
  static const bool on = std::getenv("MDH_T4_TRACE") && std::getenv("MDH_T4_TRACE")[0] == '1';
  if (!on) return nullptr;
  if (units > g_trace_units) {
    if (g_trace) cudaFree(g_trace);
    if (cudaMalloc(&g_trace, ((size_t)units * 8 + 1024) * sizeof(unsigned long long)) != cudaSuccess) {
      cudaGetLastError();
      g_trace = nullptr;
      g_trace_units = 0;
      return nullptr;
    }
    g_trace_units = units;
  }
  cudaMemset(g_trace, 0, ((size_t)g_trace_units * 8 + 1024) * sizeof(unsigned long long));
  g_trace_used = units;
  return g_trace;
}

// 2-D bf16 tensor map: inner dim `inner` (unit stride), outer dim `outer` with stride ld
static mdh_status make_map(CUtensorMap* map, const void* base, int64_t inner, int64_t outer, int64_t ld, uint32_t box_in,
                           uint32_t box_out) {
  auto fn = encode_fn();
  if (!fn) { set_error("cuTensorMapEncodeTiled unavailable (driver too old?)"); return MDH_ERR_CUDA; }
  cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)std::max<int64_t>(outer, 1)};
  cuuint64_t strides[1] = {(cuuint64_t)(std::max<int64_t>(ld, inner) * 2)};
  cuuint32_t box[2] = {box_in, box_out};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { set_error("cuTensorMapEncodeTiled failed (%d)", (int)r); return MDH_ERR_CUDA; }
  return MDH_OK;
}

static mdh_status launch_xfold(const t4::Params& P, int sms, cudaStream_t st) {
  if (!P.xfold) return MDH_OK;
  const int64_t work = (int64_t)(P.nunits / P.ssplit) * t4::BM * t4::BN / 4;
  const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>((work + 255) / 256, (int64_t)sms * 8));
  // programmatic dependent launch: the fold's launch overlaps the GEMM's tail
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(g);
  cfg.blockDim = dim3(256);
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  MDH_CUDA(cudaLaunchKernelEx(&cfg, t4::t4_xfold_kernel, P));
  return post_launch("t4_xfold_kernel");
}

static mdh_status run_permute(const t4::Layout2D& L, const uint16_t* src, char* ws, const int64_t* offMN,
                              const int64_t* offK, int64_t MN, int64_t K, cudaStream_t st, const uint16_t** out) {
  t4::PermParams Q;
  Q.src = src;
  Q.dst = (uint16_t*)(ws + L.ws_off);
  Q.ld = L.ld;
  Q.chunked = L.chunked;
  if (L.mn_major) { Q.offO = offK; Q.offI = offMN; Q.nO = K; Q.nI = MN; }
  else { Q.offO = offMN; Q.offI = offK; Q.nO = MN; Q.nI = K; }
  if (Q.chunked && Q.nI / 8 >= 32 && Q.nI / 8 < INT32_MAX) {
    const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>((Q.nO + 7) / 8, 148LL * 16));
    t4::permute_warp_kernel<<<g, 256, 0, st>>>(Q);
    *out = Q.dst;
    return post_launch("t4_permute_warp_kernel");
  }
  if (Q.chunked && Q.nO <= 65535 && Q.nI / 8 >= 4096) {   // long rows only: measured slower on MCC rows (576 chunks)
    // block sized to the row: ceil(nc/2) threads (multiple of 32, ≤ 256), two chunks each
    const int64_t nc = Q.nI / 8;
    const int tb = (int)std::min<int64_t>(256, std::max<int64_t>(32, ((nc + 1) / 2 + 31) / 32 * 32));
    dim3 grid((unsigned)std::max<int64_t>(1, (nc + 2 * tb - 1) / (2 * tb)), (unsigned)Q.nO);
    t4::permute_rows_kernel<<<grid, tb, 0, st>>>(Q);
    *out = Q.dst;
    return post_launch("t4_permute_rows_kernel");
  }
  const int64_t work = Q.chunked ? Q.nO * (Q.nI / 8) : Q.nO * Q.nI;
  const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>((work + 255) / 256, 148LL * 32));
  t4::permute_kernel<<<g, 256, 0, st>>>(Q);
  *out = Q.dst;
  return post_launch("t4_permute_kernel");
}

mdh_status launch_t4(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st) {
  if (p.t4_variant == 1024) return launch_t4_conv(p, in, out, st);
  const char* dc = nullptr;
  MDH_TRY(device_consts(p, &dc));
  const T4State* s = (const T4State*)p.tmaps;
  const Contraction& c = p.con;
  t4::Params P = s->P;
  P.C = (float*)out[0];
  P.cM = (const int64_t*)(dc + p.tab_off[4]);
  P.cN = (const int64_t*)(dc + p.tab_off[5]);
  const uint16_t* A = (const uint16_t*)in[c.a_buf] + p.in[c.a_buf].acc[0].base;
  const uint16_t* B = (const uint16_t*)in[c.b_buf] + p.in[c.b_buf].acc[0].base;
  if (s->a.permuted)
    MDH_TRY(run_permute(s->a, A, (char*)ws, (const int64_t*)(dc + p.tab_off[0]), (const int64_t*)(dc + p.tab_off[1]),
                        c.M, c.K, st, &A));
  if (s->b.permuted)
    MDH_TRY(run_permute(s->b, B, (char*)ws, (const int64_t*)(dc + p.tab_off[2]), (const int64_t*)(dc + p.tab_off[3]),
                        c.N, c.K, st, &B));
  CUtensorMap ma, mb;
  if (P.a_box) {
    auto fn = encode_fn();
    if (!fn) { set_error("cuTensorMapEncodeTiled unavailable"); return MDH_ERR_CUDA; }
    cuuint32_t estr[5] = {1, 1, 1, 1, 1};
    cuuint64_t dims[5], strides[4];
    cuuint32_t box[5];
    for (int j = 0; j < s->brank; ++j) {
      dims[j] = s->bdims[j];
      box[j] = s->bbox[j];
      if (j > 0) strides[j - 1] = s->bstrides[j - 1];
    }
    CUresult r = fn(&ma, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, (cuuint32_t)s->brank, const_cast<void*>(in[c.a_buf]), dims,
                    strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                    CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) { set_error("cuTensorMapEncodeTiled (implicit GEMM) failed (%d)", (int)r); return MDH_ERR_CUDA; }
  } else if (s->ic) {
    if ((uintptr_t)A % 16) { set_error("T4 im2col: A buffer not 16-byte aligned"); return MDH_ERR_INVALID_ARG; }
    MDH_TRY(make_im2col_map(&ma, A, *s));
  } else if (s->ag) {
    if ((uintptr_t)A % 16) { set_error("T4 gather: A buffer not 16-byte aligned"); return MDH_ERR_INVALID_ARG; }
    P.Ag = A;
    P.aM = (const int64_t*)(dc + p.tab_off[0]);
    P.aK = (const int64_t*)(dc + p.tab_off[1]);
  } else if (s->a.mn_major) MDH_TRY(make_map(&ma, A, c.M, c.K, s->a.ld, 64, 64));
  else MDH_TRY(make_map(&ma, A, c.K, c.M, s->a.ld, 64, 128));
  if (s->b.mn_major) MDH_TRY(make_map(&mb, B, c.N, c.K, s->b.ld, 64, 64));
  else MDH_TRY(make_map(&mb, B, c.K, c.N, s->b.ld, 64, s->cg == 2 ? (s->cl == 4 ? 64 : 128) : (uint32_t)P.bn));
  if (s->ag) ma = mb;
  static std::once_flag attr_once;
  static cudaError_t attr_err = cudaSuccess;
  std::call_once(attr_once, [] {
    const void* ks[5] = {(const void*)t4::gemm_kernel<0, false>, (const void*)t4::gemm_kernel<1, false>,
                         (const void*)t4::gemm_kernel<1, true>, (const void*)t4::gemm_kernel<2, false>,
                         (const void*)t4::gemm_kernel<2, true>};
    for (const void* k : ks) {
      cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, t4::SMEM_BYTES);
      if (e != cudaSuccess) attr_err = e;
    }
    const void* kg[5] = {(const void*)t4::gemm_kernel<0, false, true>, (const void*)t4::gemm_kernel<1, false, true>,
                         (const void*)t4::gemm_kernel<1, true, true>, (const void*)t4::gemm_kernel<2, false, true>,
                         (const void*)t4::gemm_kernel<2, true, true>};
    for (const void* k : kg) {
      cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, t4::SMEM_AG_BYTES);
      if (e != cudaSuccess) attr_err = e;
    }
    {
      cudaError_t e = cudaFuncSetAttribute((const void*)t4::gemm_kernel<3, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           (int)(t4::SMEM_LIMIT - t4::BN * sizeof(int64_t)));
      if (e != cudaSuccess) attr_err = e;
    }
    const void* k2[] = {(const void*)t4::gemm2_kernel<true, 2>, (const void*)t4::gemm2_kernel<true, 4>,
                        (const void*)t4::gemm2_kernel<true, 2, 512>, (const void*)t4::gemm2_kernel<true, 2, 512, 4>,
                        (const void*)t4::gemm2_kernel<true, 2, 256, t4::S2W, true>,
                        (const void*)t4::gemm2_kernel<true, 2, 512, 3, true>,
                        (const void*)t4::gemm2_kernel<true, 2, 512, 4, true>};
    for (const void* k : k2) {
      cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, t4::SMEM2_BYTES);
      if (e != cudaSuccess) attr_err = e;
    }

  });
  MDH_CUDA(attr_err);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (s->cg == 2) {
    // stream-K hybrid: with T pair-tiles on C pairs and T mod C ≠ 0, the
    // first ⌊T/C⌋ waves run whole tiles and the (tile, k-block) space of the last, partial
    // wave is split evenly over the pairs (ranges of at least SK_MIN_SEG k-blocks); tile
    // knob split=1 keeps whole tiles only
    const int CL = s->cl, NPP = CL / 2;
    // the persistent grid must be co-resident (stream-K finishers wait on other clusters):
    // at most the number of CL-CTA clusters the GPCs can hold at once (for CL = 4 fewer
    // than sms/4 when a GPC's SM count is not a multiple of 4)
    static int max_clusters[5] = {0, 0, 0, 0, 0};
    if (max_clusters[CL] == 0) {
      cudaLaunchConfig_t cfg = {};
      cudaLaunchAttribute attr[1];
      cfg.gridDim = dim3(CL * (sms / CL), 1, 1);
      cfg.blockDim = dim3(t4::THREADS, 1, 1);
      cfg.dynamicSmemBytes = t4::SMEM2_BYTES;
      attr[0].id = cudaLaunchAttributeClusterDimension;
      attr[0].val.clusterDim.x = CL;
      attr[0].val.clusterDim.y = 1;
      attr[0].val.clusterDim.z = 1;
      cfg.attrs = attr;
      cfg.numAttrs = 1;
      int n = 0;
      const cudaError_t e = CL == 4 ? cudaOccupancyMaxActiveClusters(&n, (const void*)t4::gemm2_kernel<true, 4>, &cfg)
                                    : cudaOccupancyMaxActiveClusters(&n, (const void*)t4::gemm2_kernel<true, 2>, &cfg);
      if (e != cudaSuccess || n <= 0) {
        cudaGetLastError();
        n = sms / CL;
      }
      max_clusters[CL] = std::min(n, sms / CL);
      if (std::getenv("MDH_T4_TRACE")) fprintf(stderr, "[t4] CL=%d: %d co-resident clusters (occupancy query %d)\n", CL, max_clusters[CL], (int)e);
    }
    const int C = std::max(1, max_clusters[CL]);
    const int T = P.num_tiles, R = T / C;
    P.nfull = T;
    P.sk_pairs = 0;
    P.sk_w = 0;
    // auto: stream-K only for a single partial wave of deep tiles (MCC conv5_1: 49 wide tiles
    // of 72 k-blocks on 74 pairs, 63.5 vs 66.3 µs); with more waves or shallow tiles the
    // fixups cost more than the balance gains (4096³ wide 108.8 vs 106.6 µs, 2048³ narrow
    // 32.7 vs 24.6 µs; tools/sweep_tiles.py).  Tile knob split=1 never, split≥2 whenever
    // the last wave is partial.
    const bool sk_auto = T < C && P.num_kb >= 64;
    if (s->sk_ok && T % C != 0 && (p.tiles.split >= 2 || (p.tiles.split == 0 && sk_auto))) {
      // every complete wave runs whole tiles (their epilogues overlap later MMAs); only the
      // partial last wave is spread over all pairs, so few outputs are written at the end
      const int nfull = R * C;
      const int64_t W = (int64_t)(T - nfull) * P.num_kb;
      const int sp = (int)std::min<int64_t>(std::min(C, t4::SK_MAX_PAIRS / NPP), W / t4::SK_MIN_SEG);
      if (sp >= 2) {
        P.nfull = nfull;
        P.sk_pairs = sp;
        P.sk_w = W;
        P.skpart = (float*)((char*)ws + s->tail_off);
        P.skflag = (unsigned*)((char*)ws + s->tail_off + (size_t)t4::SK_MAX_PAIRS * (s->nw / 256) * 65536 * sizeof(float));
      }
    }
    // column-unit stream (wide pair tiles; tile knob nstream=1): every pair gets an equal
    // share of 128-column units, whole K — balance without stream-K's partial-sum fixup
    P.areuse = s->nw == 512 && p.tiles.areuse != 0;
    P.vmode = 0;
    if (s->nw == 512 && CL == 2 && (p.tiles.nstream == 1 || (p.tiles.nstream == 2 && T > C && T % C != 0))) {
      // nstream=2: the complete waves run whole tiles, only the partial last wave is cut
      // into column units (no partial sums: every piece runs the whole K)
      P.vmode = 1;
      P.sk_pairs = 0;
      P.nfull = p.tiles.nstream == 2 ? (T / C) * C : 0;
      P.ups = (int)((P.N + 127) / 128);
      P.vunits = (int64_t)P.tiles_m * P.ups;
      P.idesc128 = (P.idesc & ~(0x3Fu << 17)) | ((uint32_t)(128 >> 3) << 17);
    }
    const int clusters = P.vmode ? (int)std::min<int64_t>(C, P.vunits)
                                 : (P.sk_pairs > 0 ? C : std::max(1, std::min(T, C)));
    P.trace_n = clusters * NPP * (T / clusters + 4);
    P.trace = t4_trace_buffer(P.trace_n);
    if (!P.trace) P.trace_n = 0;
    const int grid2 = CL * clusters;
    P.c_vec4 = P.c_rowmajor && P.ldc % 4 == 0 && P.cbase % 4 == 0 && (uintptr_t)P.C % 16 == 0 && P.M < INT32_MAX &&
               P.N < INT32_MAX;
    CUtensorMap mc;
    memset(&mc, 0, sizeof(mc));
    if (P.c_vec4) {
      auto fn = encode_fn();
      if (!fn) { set_error("cuTensorMapEncodeTiled unavailable (driver too old?)"); return MDH_ERR_CUDA; }
      cuuint64_t dims[2] = {(cuuint64_t)P.N, (cuuint64_t)P.M};
      cuuint64_t strides[1] = {(cuuint64_t)P.ldc * 4};
      cuuint32_t box[2] = {32, 32};
      cuuint32_t estr[2] = {1, 1};
      CUresult r = fn(&mc, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)(P.C + P.cbase), dims, strides, box, estr,
                      CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                      CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) { set_error("cuTensorMapEncodeTiled (C store map) failed (%d)", (int)r); return MDH_ERR_CUDA; }
    }
    // whole tiles only: the lean instance (no stream-K / column-unit / trace code)
    const bool lean = P.sk_pairs == 0 && !P.vmode && !P.trace && CL == 2 && P.c_vec4;
    if (lean && s->nw == 512 && s->wst == 4)
      t4::gemm2_kernel<true, 2, 512, 4, true><<<grid2, t4::THREADS, t4::SMEM2_BYTES, st>>>(ma, mb, mc, P);
    else if (lean && s->nw == 512)
      t4::gemm2_kernel<true, 2, 512, 3, true><<<grid2, t4::THREADS, t4::SMEM2_BYTES, st>>>(ma, mb, mc, P);
    else if (lean)
      t4::gemm2_kernel<true, 2, 256, t4::S2W, true><<<grid2, t4::THREADS, t4::SMEM2_BYTES, st>>>(ma, mb, mc, P);
    else if (s->nw == 512 && s->wst == 4)
      t4::gemm2_kernel<true, 2, 512, 4><<<grid2, t4::THREADS, t4::SMEM2_BYTES, st>>>(ma, mb, mc, P);
    else if (s->nw == 512) t4::gemm2_kernel<true, 2, 512><<<grid2, t4::THREADS, t4::SMEM2_BYTES, st>>>(ma, mb, mc, P);
    else if (CL == 4) t4::gemm2_kernel<true, 4><<<grid2, t4::THREADS, t4::SMEM2_BYTES, st>>>(ma, mb, mc, P);
    else t4::gemm2_kernel<true, 2><<<grid2, t4::THREADS, t4::SMEM2_BYTES, st>>>(ma, mb, mc, P);
    return post_launch("t4_gemm2_kernel");
  }
  int grid = std::min(P.num_tiles, sms);
  if (s->tail_parts) {
    grid = s->grid1;
    P.part = (float*)((char*)ws + s->tail_off);
    P.tail_cnt = (unsigned*)((char*)ws + s->tail_off + (size_t)s->tail_parts * t4::BM * t4::BN * sizeof(float));
  }
  // EPI 2 needs a 32-byte (fp32) / 16-byte (bf16) aligned output base
  const bool epi2 = s->epi == 2 && (uintptr_t)P.C % (P.out_bf16 || P.run4 ? 16 : 32) == 0;
  if (s->ag) {
    P.ag_lag = 2;   // measured on MCC conv5_1: lag 1 / 2 / 3 → 89 / 83 / 130 µs
    constexpr int TG = t4::THREADS + t4::AG_THREADS;
    if (P.c_rowmajor && !P.out_bf16) t4::gemm_kernel<0, false, true><<<grid, TG, t4::SMEM_AG_BYTES, st>>>(ma, mb, P);
    else if (epi2 && !P.out_bf16) t4::gemm_kernel<2, false, true><<<grid, TG, t4::SMEM_AG_BYTES, st>>>(ma, mb, P);
    else if (epi2) t4::gemm_kernel<2, true, true><<<grid, TG, t4::SMEM_AG_BYTES, st>>>(ma, mb, P);
    else if (!P.out_bf16) t4::gemm_kernel<1, false, true><<<grid, TG, t4::SMEM_AG_BYTES, st>>>(ma, mb, P);
    else t4::gemm_kernel<1, true, true><<<grid, TG, t4::SMEM_AG_BYTES, st>>>(ma, mb, P);
    MDH_TRY(post_launch("t4_gemm_kernel_ag"));
    return launch_xfold(P, sms, st);
  }
  if (s->epi == 3 && (uintptr_t)P.C % 16 == 0) {
    t4::gemm_kernel<3, false><<<grid, t4::THREADS, s->smem3, st>>>(ma, mb, P);
    return post_launch("t4_gemm_kernel_bulk");
  }
  if (s->epi == 3) {          // unaligned output base: the per-element scatter with 256-wide tiles
    set_error("T4 bulk-run epilogue: output base not 16-byte aligned");
    return MDH_ERR_INVALID_ARG;
  }
  if (P.c_rowmajor && !P.out_bf16) t4::gemm_kernel<0, false><<<grid, t4::THREADS, t4::SMEM_BYTES, st>>>(ma, mb, P);
  else if (epi2 && !P.out_bf16) t4::gemm_kernel<2, false><<<grid, t4::THREADS, t4::SMEM_BYTES, st>>>(ma, mb, P);
  else if (epi2) t4::gemm_kernel<2, true><<<grid, t4::THREADS, t4::SMEM_BYTES, st>>>(ma, mb, P);
  else if (!P.out_bf16) t4::gemm_kernel<1, false><<<grid, t4::THREADS, t4::SMEM_BYTES, st>>>(ma, mb, P);
  else t4::gemm_kernel<1, true><<<grid, t4::THREADS, t4::SMEM_BYTES, st>>>(ma, mb, P);
  MDH_TRY(post_launch("t4_gemm_kernel"));
  return launch_xfold(P, sms, st);
}

}  // namespace mdh

extern "C" int64_t mdh_debug_t4_trace(uint64_t* host, int64_t max_units) {
  if (!mdh::g_trace || !host) return 0;
  const int64_t n = std::min<int64_t>(max_units, mdh::g_trace_used);
  if (cudaDeviceSynchronize() != cudaSuccess ||
      cudaMemcpy(host, mdh::g_trace, (size_t)n * 8 * sizeof(uint64_t), cudaMemcpyDeviceToHost) != cudaSuccess) {
    cudaGetLastError();
    return -1;
  }
  if (n == mdh::g_trace_used &&
      cudaMemcpy(host + 8 * n, mdh::g_trace + 8 * n, 1024 * sizeof(uint64_t), cudaMemcpyDeviceToHost) != cudaSuccess) {
    cudaGetLastError();
    return -1;
  }
  return n;
}
