// t4_conv.cu — T4 "small-K" variant: a bf16 contraction whose A operand is R_out runs of L
// contiguous elements per row (an im2col row of a convolution with few input channels, e.g.
// the ResNet-50 conv1 layer of Fig 3 "MCC Inp.2", reading C-21: img[n, 2p+r, 2q+s, c]
// with C = 3, so a row is 7 runs of S·C = 21 bf16), f = MUL, ⊗ = pw(add) (Listing 12,
// P:401-429).  K = 147 is far too shallow for the TMA-fed GEMM (a 42-byte run is neither a
// TMA box nor 16-byte aligned), and the layer is bound by its 822 MB fp32 output, not by
// the tensor cores — so the kernel is built around streaming the output:
//
//   warp 12      — producer: per 128-row tile, ONE cp.async.bulk of the contiguous input
//                  span the tile's windows cover (≤ 32 KB; conv1: 9 image rows, 12.4 KB)
//                  into a 2-slot shared-memory ring (mbarrier complete_tx);
//   warps 0-7    — A builders (two groups of four warps on alternate tiles): thread t builds
//                  A row t of the tile straight from the staged
//                  span — each run is W = ⌈L/2⌉ 4-byte words (every run starts on an even
//                  element, checked at plan time), the odd tail half zeroed — and writes it
//                  with tcgen05.st into TMEM (K-major A-in-TMEM, lane = row, 2 bf16 per
//                  column; run r at columns r·W, so the K order is (run, 2W) with zero pads);
//   warp 13      — MMA issuer: tcgen05.mma.cta_group::1.kind::f16 with A from TMEM and B
//                  (the whole zero-padded filter, resident in 128B-swizzled shared memory)
//                  from a UMMA descriptor, ⌈R_out·W/8⌉ MMAs of K = 16 per tile into a
//                  double-buffered TMEM accumulator;
//   warps 8-11   — epilogue: tcgen05.ld 32x32b.x32 → 128B-swizzled 32×32 fp32 boxes →
//                  TMA tensor stores of the row-major [M, N] output (rows ≥ M clipped).
//
// The A rows never exist in HBM or in a gather buffer; HBM sees the input once (L2 catches
// the vertical window overlap) and the output once.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <mutex>
#include <vector>

#include "kcommon.cuh"

namespace mdh {
namespace t4c {

constexpr int THREADS = 448;          // 8 builder + 4 epilogue + producer + MMA warps
constexpr int BM = 128;
constexpr int STG_BYTES = 106496;     // staging ring (nslot slots of slot_bytes; conv1: 8 × 13 KB)
constexpr int MAXSLOT = 8;
constexpr int MAXR = 16;              // runs per A row
constexpr uint32_t TMEM_COLS = 512;   // D0 0, D1 128, A0 256, A1 384

struct Params {
  const uint16_t* img;                // A buffer (element 0)
  const uint16_t* flt;                // B buffer (element 0)
  const int64_t* brow;                // [N] B row offsets (B base included)
  int64_t M;
  int nmd;
  int64_t msize[3], mco[3];           // M dims, row-major (last fastest), A coefficients
  uint32_t mmul[3], mshr[3];          // i / msize[d] = umulhi(i, mmul[d]) >> mshr[d] (i < 2^30)
  int nslot, slot_bytes;              // staging ring (slot_bytes multiple of 1024, ≤ 8 slots)
  int64_t abase;
  int64_t roff[MAXR], boff[MAXR];     // run r: A / B element offset
  int64_t rmin, rmax;
  int L;                              // run length (elements)
  int num_tiles;
  uint32_t idesc;
};

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
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_load(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
// UMMA smem descriptor, K-major SWIZZLE_128B (8-row atoms of 128-byte rows, SBO 1024)
__device__ __forceinline__ uint64_t sdesc(uint32_t addr) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)(16 >> 4) << 16) | ((uint64_t)(1024 >> 4) << 32) | (1ull << 46) |
         (2ull << 61);
}
// D[tmem] (+)= A[tmem] · B[smem]
__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
      "r"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void mma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t* v) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr), "r"(v[0]),
               "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
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
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"((uint64_t)map), "r"(src),
               "r"(c0), "r"(c1)
               : "memory");
}

// element offset of A row m (its first run at r = 0 before roff)
// (32-bit index arithmetic with multiply-shift division, verified on the host for every
// index < M; the plan requires M < 2^30)
__device__ __forceinline__ int64_t a_row(const Params& P, int64_t m64) {
  int64_t off = P.abase;
  uint32_t m = (uint32_t)m64;
  for (int d = P.nmd - 1; d >= 0; --d) {
    const uint32_t q = __umulhi(m, P.mmul[d]) >> P.mshr[d];
    off += (int64_t)(m - q * (uint32_t)P.msize[d]) * P.mco[d];
    m = q;
  }
  return off;
}
// the staged span of tile t: [lo, lo + n) elements, lo 8-aligned (16 bytes)
__device__ __forceinline__ int64_t span_lo(const Params& P, int t) { return (a_row(P, (int64_t)t * BM) + P.rmin) & ~7ll; }

template <int RUNS, int W, int N>
__global__ void __launch_bounds__(THREADS, 1)
    conv_kernel(const __grid_constant__ Params P, const __grid_constant__ CUtensorMap cmap) {
  constexpr int AC = (RUNS * W + 7) / 8 * 8;    // A columns (2 bf16 each) = 8 per MMA k-step
  constexpr int KT = AC / 8;                    // MMA k-steps of 16
  constexpr int KB = (2 * AC + 63) / 64;        // B k-blocks of 64 elements
  static_assert(AC <= 128 && N <= 64 && N % 32 == 0, "TMEM plan: D 2×128, A 2×128 columns; epilogue 2 boxes");
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // (aligned by offsetting the __shared__ array itself, so every access stays LDS/STS)
  uint8_t* sm = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sB = sm;                             // KB × N rows × 128 B (SWIZZLE_128B K-major)
  uint8_t* sS = sB + KB * N * 128;              // 2 staging slots
  uint8_t* sE = sS + STG_BYTES;                 // epilogue: 4 warps × 2 buffers × 2 boxes × 4 KB
  uint64_t* bars = (uint64_t*)(sE + 16 * 4096);  // stg_full[8], stg_empty[8], a_full[2], a_empty[2], d_full[2], d_empty[2]
  int64_t* slot_lo = (int64_t*)(bars + 2 * MAXSLOT + 8);   // staged span start per slot
  uint32_t* tslot = (uint32_t*)(slot_lo + MAXSLOT);
  const uint32_t b_stg_full = smem_u32(bars), b_stg_empty = smem_u32(bars + MAXSLOT),
                 b_a_full = smem_u32(bars + 2 * MAXSLOT), b_a_empty = smem_u32(bars + 2 * MAXSLOT + 2),
                 b_d_full = smem_u32(bars + 2 * MAXSLOT + 4), b_d_empty = smem_u32(bars + 2 * MAXSLOT + 6);
  const int NS = P.nslot;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  // B: the zero-padded filter, K order (run r, element j < 2W), resident for the kernel
  // (one 16-byte chunk of 8 elements per step, its loads issued together)
  for (int e = threadIdx.x; e < N * KB * 8; e += THREADS) {
    const int n = e / (KB * 8), kc = e % (KB * 8);
    const int64_t row = P.brow[n];
    uint32_t v[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int k = kc * 8 + i, r = k / (2 * W), j = k % (2 * W);
      v[i] = (r < RUNS && j < P.L) ? __ldg(P.flt + row + P.boff[r] + j) : 0u;
    }
    const int kk = (kc & 7) * 8;
    *(uint4*)(sB + ((kc >> 3) * N + n) * 128 + (((kk >> 3) ^ (n & 7)) << 4)) =
        make_uint4(v[0] | v[1] << 16, v[2] | v[3] << 16, v[4] | v[5] << 16, v[6] | v[7] << 16);
  }
  if (threadIdx.x == 0) {
    for (int b = 0; b < NS; ++b) {
      mbar_init(b_stg_full + 8 * b, 1);
      mbar_init(b_stg_empty + 8 * b, 128);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(b_a_full + 8 * b, 128);
      mbar_init(b_a_empty + 8 * b, 1);
      mbar_init(b_d_full + 8 * b, 1);
      mbar_init(b_d_empty + 8 * b, 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 13) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tslot)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // B visible to the tensor core
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;

  if (warp == 12) {
    // ---------------- producer: one bulk copy of the tile's input span per tile
    if (lane == 0) {
      int s = 0, u = 0;                 // slot, use count of the slot ring
      for (int it = 0, t = blockIdx.x; t < P.num_tiles; ++it, t += gridDim.x) {
        if (it >= NS) mbar_wait(b_stg_empty + 8 * s, (u - 1) & 1);
        const int64_t lo = span_lo(P, t);
        const int64_t ml = min((int64_t)t * BM + BM - 1, P.M - 1);
        const int64_t hi = (a_row(P, ml) + P.rmax + P.L + 7) & ~7ll;
        const uint32_t bytes = (uint32_t)((hi - lo) * 2);
        slot_lo[s] = lo;
        mbar_expect_tx(b_stg_full + 8 * s, bytes);
        bulk_load(smem_u32(sS + s * P.slot_bytes), P.img + lo, bytes, b_stg_full + 8 * s);
        if (++s == NS) { s = 0; ++u; }
      }
    }
  } else if (warp == 13) {
    // ---------------- MMA issuer
    if (lane == 0) {
      const uint32_t b0 = smem_u32(sB);
      for (int it = 0, t = blockIdx.x; t < P.num_tiles; ++it, t += gridDim.x) {
        const int ab = it & 1;
        mbar_wait(b_a_full + 8 * ab, (it >> 1) & 1);
        if (it >= 2) mbar_wait(b_d_empty + 8 * ab, ((it >> 1) - 1) & 1);
        tc_fence_after();
        const uint32_t d = tmem + 128u * ab, a = tmem + 256u + 128u * ab;
#pragma unroll
        for (int k = 0; k < KT; ++k)
          mma_ts(d, a + 8u * k, sdesc(b0 + (k >> 2) * N * 128 + (k & 3) * 32), P.idesc, k > 0 ? 1u : 0u);
        mma_commit(b_a_empty + 8 * ab);
        mma_commit(b_d_full + 8 * ab);
      }
    }
  } else if (warp < 8) {
    // ---------------- A builders: thread = A row of the tile; two groups of four warps
    // (one per TMEM lane quarter) take alternate tiles, group g the tiles it ≡ g (mod 2),
    // so each group has two tiles' time per tile and A buffer g is always group g's
    const int g = warp >> 2, wq = warp & 3;
    const uint32_t lanes = (uint32_t)(32 * wq) << 16;
    for (int it = g, t = blockIdx.x + g * gridDim.x; t < P.num_tiles; it += 2, t += 2 * gridDim.x) {
      const int ab = g, s = it % NS, u = it / NS;
      const int64_t m = (int64_t)t * BM + 32 * wq + lane;
      uint32_t x[AC];
      const int64_t arow = m < P.M ? a_row(P, m) : 0;
      mbar_wait(b_stg_full + 8 * s, u & 1);
      if (m < P.M) {
        const uint8_t* src = sS + s * P.slot_bytes + (arow - slot_lo[s]) * 2;
#pragma unroll
        for (int r = 0; r < RUNS; ++r) {
          const uint32_t* q = (const uint32_t*)(src + P.roff[r] * 2);
#pragma unroll
          for (int w = 0; w < W; ++w) x[r * W + w] = q[w];
          if (P.L & 1) x[r * W + W - 1] &= 0xFFFFu;      // the element after the run
        }
      } else {
#pragma unroll
        for (int i = 0; i < RUNS * W; ++i) x[i] = 0;
      }
#pragma unroll
      for (int i = RUNS * W; i < AC; ++i) x[i] = 0;
      mbar_arrive(b_stg_empty + 8 * s);
      if (it >= 2) mbar_wait(b_a_empty + 8 * ab, ((it >> 1) - 1) & 1);
      tc_fence_after();
      const uint32_t a = tmem + lanes + 256u + 128u * ab;
#pragma unroll
      for (int c = 0; c < AC / 8; ++c) tmem_st8(a + 8u * c, x + 8 * c);
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      tc_fence_before();
      mbar_arrive(b_a_full + 8 * ab);
    }
  } else {
    // ---------------- epilogue: TMEM → swizzled 32×32 boxes → TMA tensor stores
    const int q = warp - 8;
    const uint32_t lanes = (uint32_t)(32 * q) << 16;
    for (int it = 0, t = blockIdx.x; t < P.num_tiles; ++it, t += gridDim.x) {
      const int db = it & 1;
      mbar_wait(b_d_full + 8 * db, (it >> 1) & 1);
      tc_fence_after();
      // the tile's N/32 boxes: TMEM → registers (all chunks, then free the accumulator), one
      // proxy fence for the whole tile, then one TMA store per box in one bulk group
      uint32_t v[N / 32][32];
#pragma unroll
      for (int c = 0; c < N / 32; ++c) tmem_ld32(tmem + lanes + 128u * db + 32u * c, v[c]);
      tc_fence_before();
      mbar_arrive(b_d_empty + 8 * db);
      uint8_t* box = sE + (q * 2 + (it & 1)) * 8192;    // double-buffered box pair per warp
      if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      __syncwarp();
#pragma unroll
      for (int c = 0; c < N / 32; ++c) {
        const uint32_t row = smem_u32(box + c * 4096) + lane * 128;
#pragma unroll
        for (int j = 0; j < 8; ++j)
          asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(row + ((j ^ (lane & 7)) << 4)), "r"(v[c][4 * j]),
                       "r"(v[c][4 * j + 1]), "r"(v[c][4 * j + 2]), "r"(v[c][4 * j + 3])
                       : "memory");
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) {
#pragma unroll
        for (int c = 0; c < N / 32; ++c) tma_store_2d(&cmap, smem_u32(box + c * 4096), 32 * c, t * BM + 32 * q);
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 13) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS));
  }
}

// instantiated shapes (runs, words per run, N): conv1 7×7/s2 with C = 3 (L = 21), a 3×3
// layer with C = 3 (L = 9), each with 64 output channels
struct Shape {
  int runs, w, n;
  void (*k)(Params, CUtensorMap);
};
static const Shape kShapes[] = {
    {7, 11, 64, conv_kernel<7, 11, 64>},
    {3, 5, 64, conv_kernel<3, 5, 64>},
};

static size_t smem_bytes(int runs, int w, int n) {
  const int ac = (runs * w + 7) / 8 * 8, kb = (2 * ac + 63) / 64;
  return 1024 + (size_t)kb * n * 128 + STG_BYTES + 16 * 4096 + (2 * MAXSLOT + 8) * 8 + MAXSLOT * 8 + 16;
}

// multiply-shift constants for i / d, exact for every i < limit (checked exhaustively)
static bool magic_div(uint32_t d, uint32_t limit, uint32_t* mul, uint32_t* shr) {
  for (uint32_t s = 0; s < 32; ++s) {
    const unsigned __int128 two = (unsigned __int128)1 << (32 + s);
    const unsigned __int128 m = (two + d - 1) / d;
    if (m >> 32) continue;
    bool ok = true;
    for (uint32_t i = 0; i < limit && ok; ++i)
      ok = (uint32_t)(((uint64_t)i * (uint64_t)m) >> 32 >> s) == i / d;
    if (ok) {
      *mul = (uint32_t)m;
      *shr = s;
      return true;
    }
  }
  return false;
}

}  // namespace t4c

// ---------------------------------------------------------------------------- host
// auxi layout: [0] = 0x7C (tag), [1] = shape index, [2] = output base, [3] = ldc
// tab_off[12] = brow (int64 [N]); the scalar Params live in host_const at tab_off[13]
bool prepare_t4_conv(Plan* p) {
  const Contraction& c = p->con;
  if (p->tiles.implicit != 0 && p->tiles.implicit != 5) return false;   // tile knob implicit=5 forces, others skip
  if (c.Z != 1 || c.nm < 1 || c.nm > 3 || c.nn < 1 || c.nk < 1 || p->n_out != 1) return false;
  const Buf& Ab = p->in[c.a_buf];
  const Buf& Bb = p->in[c.b_buf];
  if (Ab.dtype != MDH_BF16 || Bb.dtype != MDH_BF16 || p->out[0].dtype != MDH_F32) return false;
  if (Ab.nacc != 1 || Bb.nacc != 1 || p->out[0].nacc != 1) return false;
  const Access& A = Ab.acc[0];
  const Access& B = Bb.acc[0];
  const Access& C = p->out[0].acc[0];
  // K: the innermost K dims form a contiguous run in A and in B (same order), the rest are runs
  int inner = c.nk;           // kd[inner..nk) are run dims
  int64_t L = 1;
  while (inner > 0) {
    const int d = c.kd[inner - 1];
    if (A.L[d] != L || B.L[d] != L) break;
    L *= p->size[d];
    --inner;
  }
  if (inner == c.nk || L < 2) return false;
  int64_t runs = 1;
  for (int i = 0; i < inner; ++i) runs *= p->size[c.kd[i]];
  const int W = (int)((L + 1) / 2);
  int shape = -1;
  for (int i = 0; i < (int)(sizeof(t4c::kShapes) / sizeof(t4c::kShapes[0])); ++i)
    if (t4c::kShapes[i].runs == runs && t4c::kShapes[i].w == W && t4c::kShapes[i].n == c.N) shape = i;
  if (shape < 0) return false;
  t4c::Params P;
  memset(&P, 0, sizeof(P));
  P.L = (int)L;
  P.rmin = INT64_MAX;
  P.rmax = INT64_MIN;
  for (int64_t r = 0; r < runs; ++r) {
    int64_t rem = r, ao = 0, bo = 0;
    for (int i = inner - 1; i >= 0; --i) {
      const int d = c.kd[i];
      const int64_t v = rem % p->size[d];
      rem /= p->size[d];
      ao += v * A.L[d];
      bo += v * B.L[d];
    }
    P.roff[r] = ao;
    P.boff[r] = bo;
    P.rmin = std::min(P.rmin, ao);
    P.rmax = std::max(P.rmax, ao);
    if (ao % 2) return false;                 // runs start on 4-byte words
  }
  // M: A row offsets a_row(m) = abase + Σ i_d·mco[d], monotone in m (each coefficient at
  // least the span of the dims inside it), even
  P.nmd = c.nm;
  P.abase = A.base;
  int64_t span = 0;
  for (int i = c.nm - 1; i >= 0; --i) {
    const int d = c.md[i];
    P.msize[i] = p->size[d];
    P.mco[i] = A.L[d];
    if (A.L[d] < 0 || A.L[d] % 2 || (p->size[d] > 1 && A.L[d] <= span && span > 0)) return false;
    span += (p->size[d] - 1) * A.L[d];
  }
  if (A.base % 2 || (Ab.elems % 8) != 0) return false;
  P.M = c.M;
  if (c.M >= (1ll << 30)) return false;
  for (int i = 0; i < c.nm; ++i)
    if (P.msize[i] >= (1ll << 31)) return false;
  P.num_tiles = (int)((c.M + t4c::BM - 1) / t4c::BM);
  // i / msize[d] by multiply-shift for every quotient the kernel forms (i < M)
  for (int i = 0; i < c.nm; ++i)
    if (!t4c::magic_div((uint32_t)P.msize[i], (uint32_t)c.M, &P.mmul[i], &P.mshr[i])) return false;
  // every tile's staged span fits a slot
  auto arow = [&](int64_t m) {
    int64_t off = P.abase;
    for (int d = P.nmd - 1; d >= 0; --d) {
      off += (m % P.msize[d]) * P.mco[d];
      m /= P.msize[d];
    }
    return off;
  };
  int64_t maxspan = 0;
  for (int64_t t = 0; t < P.num_tiles; ++t) {
    const int64_t lo = (arow(t * t4c::BM) + P.rmin) & ~7ll;
    const int64_t hi = (arow(std::min(t * t4c::BM + t4c::BM - 1, c.M - 1)) + P.rmax + L + 7) & ~7ll;
    if (hi > Ab.elems) return false;
    maxspan = std::max(maxspan, (hi - lo) * 2);
  }
  // slots of the span rounded to 1 KB, as many as the ring holds (2..8; conv1: 13 KB × 4)
  P.slot_bytes = (int)((maxspan + 1023) / 1024 * 1024);
  P.nslot = std::min<int>(t4c::MAXSLOT, t4c::STG_BYTES / std::max(P.slot_bytes, 1));
  if (P.nslot < 2) return false;
  // tile knob stages: staging slots in flight (forced; default 4 — measured on conv1 N=256:
  // see DESIGN.md §6)
  const bool forced = p->tiles.source.find("forced") != std::string::npos;
  if (forced && p->tiles.stages >= 2) P.nslot = std::min(P.nslot, p->tiles.stages);
  else P.nslot = std::min(P.nslot, 4);
  // an even slot count: slot s then always serves the same builder group (tiles it ≡ s
  // mod 2), so no group can reach a slot's next use while the other group's use of it is
  // still in flight — a waiter two phases behind would alias the mbarrier parity
  P.nslot &= ~1;
  // output: row-major [M, N] fp32, 16-byte aligned rows
  int64_t ldc = 0;
  {
    // cN[n] = n (unit stride over the N group), cM[m] = m·ldc
    int64_t st = 1;
    for (int i = c.nn - 1; i >= 0; --i) {
      const int d = c.nd[i];
      if (C.L[d] != st) return false;
      st *= p->size[d];
    }
    ldc = 1;
    int64_t expect = -1;
    for (int i = c.nm - 1; i >= 0; --i) {
      const int d = c.md[i];
      if (expect < 0) { ldc = C.L[d]; expect = C.L[d]; }
      if (C.L[d] != expect) return false;
      expect *= p->size[d];
    }
    if (ldc < c.N || (ldc * 4) % 16 || (C.base * 4) % 16) return false;
  }
  // B rows
  std::vector<int64_t> brow((size_t)c.N);
  for (int64_t n = 0; n < c.N; ++n) {
    int64_t rem = n, off = B.base;
    for (int i = c.nn - 1; i >= 0; --i) {
      const int d = c.nd[i];
      off += (rem % p->size[d]) * B.L[d];
      rem /= p->size[d];
    }
    brow[(size_t)n] = off;
  }
  // instruction descriptor (kind::f16): D f32, A/B bf16, both K-major, N>>3, M>>4
  P.idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(c.N >> 3) << 17) | ((uint32_t)(t4c::BM >> 4) << 24);
  p->host_const.clear();
  p->tab_off[12] = add_const(p, brow.data(), brow.size() * sizeof(int64_t));
  p->tab_off[13] = add_const(p, &P, sizeof(P));
  p->auxi = {0x7C, shape, C.base, ldc};
  p->t4_variant = 1024;
  p->ws_kernel = 0;
  p->tiles.bm = t4c::BM;
  p->tiles.bn = (int)c.N;
  p->tiles.bk = 16;
  p->tiles.stages = P.nslot;
  p->tiles.cluster = 1;
  p->tiles.implicit = 5;
  p->why += "; small-K direct contraction (A rows built from staged runs in TMEM)";
  return true;
}

mdh_status launch_t4_conv(const Plan& p, const void* const* in, void* const* out, cudaStream_t st) {
  const char* dc = nullptr;
  MDH_TRY(device_consts(p, &dc));
  const Contraction& c = p.con;
  t4c::Params P;
  memcpy(&P, p.host_const.data() + p.tab_off[13], sizeof(P));
  P.img = (const uint16_t*)in[c.a_buf];
  P.flt = (const uint16_t*)in[c.b_buf];
  P.brow = (const int64_t*)(dc + p.tab_off[12]);
  const t4c::Shape& S = t4c::kShapes[p.auxi[1]];
  // output map: row-major [M, N] fp32 at out + cbase, row stride ldc, 32×32 boxes, 128B swizzle
  static PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      enc = (PFN_cuTensorMapEncodeTiled_v12000)f;
  });
  if (!enc) { set_error("cuTensorMapEncodeTiled unavailable"); return MDH_ERR_CUDA; }
  CUtensorMap cmap;
  cuuint64_t dims[2] = {(cuuint64_t)c.N, (cuuint64_t)c.M};
  cuuint64_t strides[1] = {(cuuint64_t)(p.auxi[3] * 4)};
  cuuint32_t box[2] = {32, 32};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(&cmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (float*)out[0] + p.auxi[2], dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { set_error("cuTensorMapEncodeTiled (conv output) failed (%d)", (int)r); return MDH_ERR_CUDA; }
  const size_t smem = t4c::smem_bytes(S.runs, S.w, S.n);
  MDH_CUDA(cudaFuncSetAttribute((const void*)S.k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int sms = 148;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, p.device) != cudaSuccess) { cudaGetLastError(); sms = 148; }
  const unsigned grid = (unsigned)std::max(1, std::min(P.num_tiles, sms));
  S.k<<<grid, t4c::THREADS, smem, st>>>(P, cmap);
  return post_launch("t4_conv_kernel");
}

}  // namespace mdh
