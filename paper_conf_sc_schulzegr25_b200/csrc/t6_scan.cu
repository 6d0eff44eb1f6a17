// t6_scan.cu — T6: the prefix-sum combine operator ps(add) (Listing 17; SURVEY
// §8(f) F1) and MBBS read as md_hom(id, (pw(add), ps(add))) (reading C-30).
//
// One ps dim d_ps is kept and folded over [0, k]; other kept (cc) dims enumerate rows c;
// pw(add) dims are folded completely.  Because every operator here is +, the result is
//   R[c, k] = Σ_{t ≤ k} z[c, t],   z[c, t] = Σ_{pw} f(x(c, t, pw))
// Deterministic throughout (every sum in a fixed association order, no float atomics).
// Three paths, chosen at plan time (prepare_t6):
//
//  * Long unit-stride rows read straight from the input (no pw dims, f = IDENTITY) — the
//    prefix sum of 2^26 fp32 — take ONE persistent streaming kernel (t6_stream_scan_kernel,
//    the default): two CTAs per SM each own a slice of every segment, brought into a shared-
//    memory ring by TMA bulk copies issued three jobs ahead; each CTA publishes its slice
//    total as a self-validating (tag, value) word, and its exclusive prefix is the carry
//    plus the totals of the lower CTAs in CTA order (polled by warp 0, no grid barrier);
//    the slice is scanned in place (per-thread sequential runs, warp/CTA scans in order)
//    and written back with a bulk store — HBM sees one read and one write per element.
//    (t6_seg_scan_kernel, a segmented variant with a grid barrier between a reduce and a
//    re-scan pass, stays behind tile knob seg > 0 for measurements.)
//  * One pw dim folded into a unit-stride ps dim in fp32 (MBBS) — the column fold
//    (t6_colfold_kernel: 4 columns per thread with 16-byte loads, the rows split over
//    blocks × 8 threads, folded in order by a per-column-group ticket), then the register
//    row scan t6_rowscan4_kernel launched as a programmatic dependent (rows ≤ 8 × 4096).
//  * Otherwise: K1 z[c, t] = the pw fold per (c, t) (t6_fold_kernel), K2 a block scan of
//    each 4096-element chunk with its total (t6_chunk_scan_kernel, or one 1024-thread row
//    scan for short rows), K3 an exclusive scan of the chunk totals (t6_sums_kernel), K4
//    the chunk offsets added and the result written through out_view (t6_fix_kernel).
#include <algorithm>
#include <mutex>

#include <type_traits>

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
  // tree scan: tiles per row, levels of the per-row binary tree over tiles (node offsets
  // and counts per level), nodes per row
  int64_t nt, npr;
  int nlev;
  int64_t loff[48], lcnt[48];
  void* out;
  int odt;
  void* z;        // V[Nc][T]
  void* loc;      // V[Nc][T]
  void* sums;     // V[Nc][nq]
  // column fold (fp32, one pw dim, unit stride along the ps dim): row range split over
  // S blocks × 8 threads; S > 1: per-split partials colpart[S][Nc·T] and a ticket per
  // 128-column group (zero at rest); the last block folds the splits in order
  int colS;
  float* colpart;
  unsigned* colcnt;
};

// K1 with the pw range split over threadIdx.y (blockDim.y contiguous sub-ranges, folded in
// order through shared memory): 32 consecutive (c, t) points per block row keep loads
// coalesced.  A single pw dim (MBBS's i) walks a plain stride, 8 loads in flight per
// thread, added in index order.
constexpr int T6_COL_SMAX = 32;
constexpr int64_t T6_ROW_SMEM = 48 * 1024;   // rows up to this many bytes take t6_rowscan_kernel

template <class V>
__global__ void __launch_bounds__(1024) t6_fold_kernel(const __grid_constant__ T6Params P) {
  __shared__ V part[32][32];
  const int Y = blockDim.y;
  const int64_t total = P.Nc * P.T;
  int64_t npts = 1;
  for (int q = 0; q < P.npw; ++q) npts *= P.pwsize[q];
  const int64_t per = (npts + Y - 1) / Y;
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
    if (P.npw == 1 && P.f == MDH_F_IDENTITY) {
      const int64_t L = P.Lpw[0][0];
      int64_t o = off[0] + L * r0;
      int64_t r = r0;
      acc = load_as<V>(P.ptr[0], P.dt[0], o);
      o += L;
      ++r;
      for (; r + 8 <= r1; r += 8, o += 8 * L) {
        V y[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) y[u] = load_as<V>(P.ptr[0], P.dt[0], o + u * L);
#pragma unroll
        for (int u = 0; u < 8; ++u) acc = Arith<V>::add(acc, y[u]);
      }
      for (; r < r1; ++r, o += L) acc = Arith<V>::add(acc, load_as<V>(P.ptr[0], P.dt[0], o));
    } else {
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
    }
    part[threadIdx.y][threadIdx.x] = acc;
    __syncthreads();
    if (threadIdx.y == 0 && e < total) {
      V s = part[0][threadIdx.x];
      for (int y = 1; y < Y; ++y) s = Arith<V>::add(s, part[y][threadIdx.x]);   // sub-range order
      ((V*)P.z)[e] = s;
    }
    __syncthreads();
  }
}

// K1 for MBBS-like shapes (few points, long pw range): each thread folds 4 consecutive
// columns (one 16-byte load per row, 8 rows in flight) over its share of the rows; the
// row range is split over blockIdx.y (S splits) × threadIdx.y (8), so S·(#column groups)
// blocks fill the GPU even when the points alone cannot.  Fold order: rows ascending
// inside a sub-range, sub-ranges (threadIdx.y, then blockIdx.y) ascending — fixed, so the
// result is deterministic.
__global__ void __launch_bounds__(256) t6_colfold_kernel(const __grid_constant__ T6Params P) {
  // the row scan that follows is launched with programmatic stream serialization: let it
  // be scheduled now (it waits in griddepcontrol.wait until this grid's writes are visible)
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  __shared__ float4 part[8][32];
  __shared__ int last;
  const int64_t T = P.T;
  const int64_t gpr = (T + 127) / 128;
  const int64_t c = blockIdx.x / gpr, g = blockIdx.x % gpr;
  const int64_t t = g * 128 + threadIdx.x * 4;
  const int S = gridDim.y, s = blockIdx.y;
  const int64_t npts = P.pwsize[0];
  const int64_t nsub = (int64_t)S * 8, sub = (int64_t)s * 8 + threadIdx.y;
  const int64_t per = (npts + nsub - 1) / nsub;
  const int64_t r0 = min(npts, sub * per), r1 = min(npts, r0 + per);
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  if (t < T && r0 < r1) {
    int64_t off = P.base[0] + P.Lt[0] * t, rem = c;
    for (int q = P.nrowd - 1; q >= 0; --q) {
      const int64_t v = rem % P.rowsize[q];
      rem /= P.rowsize[q];
      off += P.Lrow[0][q] * v;
    }
    const int64_t L = P.Lpw[0][0];
    const float* x = (const float*)P.ptr[0] + off + L * r0;
    acc = __ldg(reinterpret_cast<const float4*>(x));
    x += L;
    int64_t r = r0 + 1;
    for (; r + 8 <= r1; r += 8, x += 8 * L) {
      float4 y[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) y[u] = __ldg(reinterpret_cast<const float4*>(x + u * L));
#pragma unroll
      for (int u = 0; u < 8; ++u) { acc.x += y[u].x; acc.y += y[u].y; acc.z += y[u].z; acc.w += y[u].w; }
    }
    for (; r < r1; ++r, x += L) {
      const float4 y = __ldg(reinterpret_cast<const float4*>(x));
      acc.x += y.x; acc.y += y.y; acc.z += y.z; acc.w += y.w;
    }
  }
  part[threadIdx.y][threadIdx.x] = acc;
  __syncthreads();
  const int64_t e = c * T + t;
  if (threadIdx.y == 0) {
    float4 b = part[0][threadIdx.x];
    for (int y = 1; y < 8; ++y) {
      const float4 q = part[y][threadIdx.x];
      b.x += q.x; b.y += q.y; b.z += q.z; b.w += q.w;
    }
    if (t < T) {
      if (S == 1) *reinterpret_cast<float4*>((float*)P.z + e) = b;
      else *reinterpret_cast<float4*>(P.colpart + (int64_t)s * P.Nc * T + e) = b;
    }
  }
  if (S > 1) {
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0 && threadIdx.y == 0) last = atomicAdd(P.colcnt + blockIdx.x, 1u) == (unsigned)(S - 1);
    __syncthreads();
    if (!last) return;
    if (threadIdx.y == 0) {
      __threadfence();
      if (t < T) {
        float4 b = __ldcg(reinterpret_cast<const float4*>(P.colpart + e));
        for (int k = 1; k < S; ++k) {
          const float4 q = __ldcg(reinterpret_cast<const float4*>(P.colpart + (int64_t)k * P.Nc * T + e));
          b.x += q.x; b.y += q.y; b.z += q.z; b.w += q.w;
        }
        *reinterpret_cast<float4*>((float*)P.z + e) = b;
      }
      if (threadIdx.x == 0) P.colcnt[blockIdx.x] = 0u;   // back to rest for the next execute
    }
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

// Inclusive scan of short rows (T ≤ T6_ROW_MAX) of the fold result z, one block of 1024
// threads per row: the row is staged in shared memory by coalesced loads, each thread
// scans a segment of ⌈T/1024⌉ consecutive elements, segment totals are scanned by warp
// shuffles (lane order) and then across the 32 warps (warp order) — a fixed association,
// deterministic — and the result leaves through out_view with coalesced stores.
template <class V>
__global__ void __launch_bounds__(1024) t6_rowscan_kernel(const __grid_constant__ T6Params P) {
  extern __shared__ __align__(16) unsigned char t6rs_raw[];
  V* zs = reinterpret_cast<V*>(t6rs_raw);
  __shared__ V wtot[32];
  const int64_t c = blockIdx.x, T = P.T;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const V* zr = (const V*)P.z + c * T;
  for (int64_t k = tid; k < T; k += 1024) zs[k] = zr[k];
  __syncthreads();
  const int64_t seg = (T + 1023) / 1024;
  const int64_t a0 = min(T, tid * seg), a1 = min(T, a0 + seg);
  V sum = (V)0;
  for (int64_t k = a0; k < a1; ++k) sum = Arith<V>::add(sum, zs[k]);
  V incl = sum;                                   // inclusive scan over the lanes
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const V y = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl = Arith<V>::add(y, incl);
  }
  V excl = __shfl_up_sync(0xffffffffu, incl, 1);
  if (lane == 0) excl = (V)0;
  if (lane == 31) wtot[wid] = incl;
  __syncthreads();
  if (wid == 0) {
    V w = wtot[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const V y = __shfl_up_sync(0xffffffffu, w, o);
      if (lane >= o) w = Arith<V>::add(y, w);
    }
    wtot[lane] = w;                               // inclusive over warps
  }
  __syncthreads();
  V run = wid > 0 ? Arith<V>::add(wtot[wid - 1], excl) : excl;   // exclusive prefix of the segment
  for (int64_t k = a0; k < a1; ++k) { run = Arith<V>::add(run, zs[k]); zs[k] = run; }
  __syncthreads();
  for (int64_t k = tid; k < T; k += 1024) store_as<V>(P.out, P.odt, t6_out_offset(P, c, k), zs[k]);
}

// The same scan for fp32 rows of T = 1024·4·nv elements (nv ≤ 8) and a contiguous, 16-byte
// aligned fp32 output row: each thread's segment of T/1024 consecutive elements is held in
// registers (float4 loads from the fold result, float4 stores to out) — no shared-memory
// staging — with exactly the association of t6_rowscan_kernel (bit-identical results).
// Launched as a programmatic dependent of the column fold: griddepcontrol.wait returns once
// the fold grid has completed and its writes are visible.
__global__ void __launch_bounds__(1024) t6_rowscan4_kernel(const __grid_constant__ T6Params P) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  __shared__ float wtot[32];
  const int64_t c = blockIdx.x, T = P.T;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int nv = (int)(T / 4096);
  const float4* zr = reinterpret_cast<const float4*>((const float*)P.z + c * T) + (int64_t)tid * nv;
  float4 v[8];
#pragma unroll
  for (int q = 0; q < 8; ++q)
    if (q < nv) v[q] = __ldcg(zr + q);
  float sum = 0.f;
#pragma unroll
  for (int q = 0; q < 8; ++q)
    if (q < nv) { sum += v[q].x; sum += v[q].y; sum += v[q].z; sum += v[q].w; }
  float incl = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const float y = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl = y + incl;
  }
  float excl = __shfl_up_sync(0xffffffffu, incl, 1);
  if (lane == 0) excl = 0.f;
  if (lane == 31) wtot[wid] = incl;
  __syncthreads();
  if (wid == 0) {
    float w = wtot[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const float y = __shfl_up_sync(0xffffffffu, w, o);
      if (lane >= o) w = y + w;
    }
    wtot[lane] = w;
  }
  __syncthreads();
  float run = wid > 0 ? wtot[wid - 1] + excl : excl;
  float4* orow = reinterpret_cast<float4*>((float*)P.out + t6_out_offset(P, c, 0)) + (int64_t)tid * nv;
#pragma unroll
  for (int q = 0; q < 8; ++q)
    if (q < nv) {
      run += v[q].x; v[q].x = run;
      run += v[q].y; v[q].y = run;
      run += v[q].z; v[q].z = run;
      run += v[q].w; v[q].w = run;
      orow[q] = v[q];
    }
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

// ---- single-pass segmented scan (long unit-stride rows) ----------------------------
constexpr int T6S_THREADS = 256, T6S_UNIT = 1024;

__device__ __forceinline__ void t6_grid_barrier(unsigned* bar) {
  __syncthreads();
  if (threadIdx.x == 0) {
    volatile unsigned* gen = bar + 1;
    const unsigned g = *gen;
    __threadfence();
    if (atomicAdd(bar, 1u) == gridDim.x - 1) {
      bar[0] = 0u;
      __threadfence();
      atomicAdd(bar + 1, 1u);
    } else {
      while (*gen == g) __nanosleep(32);
    }
    __threadfence();
  }
  __syncthreads();
}

// Σ p[0..n) in a fixed order (lane-strided partial sums, then a fixed shuffle tree),
// computed by warp 0 and returned to every thread through `slot`
template <class V>
__device__ __forceinline__ V t6_sum_fixed(const V* p, int n, V* slot) {
  if (threadIdx.x < 32) {
    V a = (V)0;
    for (int i = threadIdx.x; i < n; i += 32) a = Arith<V>::add(a, *((volatile const V*)(p + i)));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) a = Arith<V>::add(a, __shfl_down_sync(0xffffffffu, a, o));
    if (threadIdx.x == 0) *slot = a;
  }
  __syncthreads();
  const V r = *slot;
  __syncthreads();
  return r;
}

template <class V>
__device__ __forceinline__ V t6_block_sum(V a, V* red) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) a = Arith<V>::add(a, __shfl_down_sync(0xffffffffu, a, o));
  if (lane == 0) red[warp] = a;
  __syncthreads();
  V t = red[0];
  for (int w = 1; w < T6S_THREADS / 32; ++w) t = Arith<V>::add(t, red[w]);
  __syncthreads();
  return t;
}

template <class V>
__global__ void __launch_bounds__(T6S_THREADS, 3) t6_seg_scan_kernel(const __grid_constant__ T6Params P) {
  constexpr int VEC = 16 / sizeof(V);
  constexpr int PER = T6_CHUNK / T6S_THREADS;            // 16 elements per thread per tile
  __shared__ __align__(16) V tile[T6_CHUNK + T6_CHUNK / 32];
  __shared__ V red[T6S_THREADS / 32];
  __shared__ V slot;
  const int G = gridDim.x, b = blockIdx.x, tid = threadIdx.x;
  const int lane = tid & 31, warp = tid >> 5;
  V* part = (V*)P.sums;                                   // [2][G] CTA totals per segment
  unsigned* bar = (unsigned*)P.loc;
  const V* X = (const V*)P.ptr[0];
  V* Y = (V*)P.out;
  int buf = 0;
  for (int64_t c = 0; c < P.Nc; ++c) {
    int64_t xrow = P.base[0], rem = c;
    for (int d = P.nrowd - 1; d >= 0; --d) {
      const int64_t v = rem % P.rowsize[d];
      rem /= P.rowsize[d];
      xrow += P.Lrow[0][d] * v;
    }
    const int64_t orow = t6_out_offset(P, c, 0);
    const bool vx = ((xrow & (VEC - 1)) == 0) && (((uintptr_t)X & 15) == 0);
    const bool vy = ((orow & (VEC - 1)) == 0) && (((uintptr_t)Y & 15) == 0);
    V carry = (V)0;
    for (int64_t s0 = 0; s0 < P.T; s0 += P.nq) {            // nq = segment length here
      const int64_t len = min(P.nq, P.T - s0);
      const int64_t nunit = (len + T6S_UNIT - 1) / T6S_UNIT;
      const int64_t e0 = s0 + min(len, (int64_t)b * nunit / G * T6S_UNIT);
      const int64_t e1 = s0 + min(len, (int64_t)(b + 1) * nunit / G * T6S_UNIT);
      // (A) reduce [e0, e1): thread-strided 16-byte vectors, fixed order
      V acc = (V)0;
      if (vx) {
        const int64_t nv = (e1 - e0) / VEC;                // e0 - s0 is a multiple of UNIT
        const uint4* xv = reinterpret_cast<const uint4*>(X + xrow + e0);
        int64_t i = tid;
        for (; i + 3 * T6S_THREADS < nv; i += 4 * T6S_THREADS) {
          uint4 q[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) q[u] = __ldg(xv + i + u * T6S_THREADS);
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const V* e = reinterpret_cast<const V*>(&q[u]);
#pragma unroll
            for (int k = 0; k < VEC; ++k) acc = Arith<V>::add(acc, e[k]);
          }
        }
        for (; i < nv; i += T6S_THREADS) {
          const uint4 q = __ldg(xv + i);
          const V* e = reinterpret_cast<const V*>(&q);
#pragma unroll
          for (int k = 0; k < VEC; ++k) acc = Arith<V>::add(acc, e[k]);
        }
        for (int64_t t = e0 + nv * VEC + tid; t < e1; t += T6S_THREADS) acc = Arith<V>::add(acc, X[xrow + t]);
      } else {
        for (int64_t t = e0 + tid; t < e1; t += T6S_THREADS) acc = Arith<V>::add(acc, X[xrow + t]);
      }
      const V tot_b = t6_block_sum<V>(acc, red);
      if (tid == 0) part[buf * G + b] = tot_b;
      t6_grid_barrier(bar);
      // (B) exclusive prefix of this CTA and the segment total, both in CTA order
      const V lower = t6_sum_fixed<V>(part + buf * G, b, &slot);
      const V segtot = t6_sum_fixed<V>(part + buf * G, G, &slot);
      V run = Arith<V>::add(carry, lower);
      // (C) re-scan [e0, e1) in 4096-element tiles (L2 hits), running carry in tile order;
      // the next full tile's vectors are loaded into registers while this one is scanned
      constexpr int NV = T6_CHUNK / VEC / T6S_THREADS;
      uint4 nxt[NV];
      if (vx && e1 - e0 >= T6_CHUNK) {
        const uint4* xv = reinterpret_cast<const uint4*>(X + xrow + e0);
#pragma unroll
        for (int k = 0; k < NV; ++k) nxt[k] = __ldg(xv + k * T6S_THREADS + tid);
      }
      for (int64_t t0 = e0; t0 < e1; t0 += T6_CHUNK) {
        const int n = (int)min((int64_t)T6_CHUNK, e1 - t0);
        if (vx && n == T6_CHUNK) {
          uint4 cur[NV];
#pragma unroll
          for (int k = 0; k < NV; ++k) cur[k] = nxt[k];
          if (e1 - t0 >= 2 * T6_CHUNK) {
            const uint4* xn = reinterpret_cast<const uint4*>(X + xrow + t0 + T6_CHUNK);
#pragma unroll
            for (int k = 0; k < NV; ++k) nxt[k] = __ldg(xn + k * T6S_THREADS + tid);
          }
#pragma unroll
          for (int k = 0; k < NV; ++k) {
            const int vi = k * T6S_THREADS + tid;
            const uint4 q = cur[k];
            const V* e = reinterpret_cast<const V*>(&q);
#pragma unroll
            for (int u = 0; u < VEC; ++u) {
              const int j = vi * VEC + u;
              tile[j + (j >> 5)] = e[u];
            }
          }
        } else {
#pragma unroll
          for (int k = 0; k < PER; ++k) {
            const int j = k * T6S_THREADS + tid;
            tile[j + (j >> 5)] = j < n ? X[xrow + t0 + j] : (V)0;
          }
        }
        __syncthreads();
        V v[PER];
        V r = (V)0;
#pragma unroll
        for (int k = 0; k < PER; ++k) {
          const int j = tid * PER + k;
          r = k == 0 ? tile[j + (j >> 5)] : Arith<V>::add(r, tile[j + (j >> 5)]);
          v[k] = r;
        }
        V incl = r;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const V nb = __shfl_up_sync(0xffffffffu, incl, o);
          if (lane >= o) incl = Arith<V>::add(nb, incl);
        }
        if (lane == 31) red[warp] = incl;
        __syncthreads();
        V base = run;
        for (int w = 0; w < warp; ++w) base = Arith<V>::add(base, red[w]);
        V tilesum = run;
        for (int w = 0; w < T6S_THREADS / 32; ++w) tilesum = Arith<V>::add(tilesum, red[w]);
        const V prev = __shfl_up_sync(0xffffffffu, incl, 1);
        const V excl = lane == 0 ? base : Arith<V>::add(base, prev);
#pragma unroll
        for (int k = 0; k < PER; ++k) {
          const int j = tid * PER + k;
          tile[j + (j >> 5)] = Arith<V>::add(excl, v[k]);
        }
        __syncthreads();
        if (vy && n == T6_CHUNK) {
          uint4* yv = reinterpret_cast<uint4*>(Y + orow + t0);
#pragma unroll
          for (int k = 0; k < T6_CHUNK / VEC / T6S_THREADS; ++k) {
            const int vi = k * T6S_THREADS + tid;
            uint4 q;
            V* e = reinterpret_cast<V*>(&q);
#pragma unroll
            for (int u = 0; u < VEC; ++u) {
              const int j = vi * VEC + u;
              e[u] = tile[j + (j >> 5)];
            }
            __stcs(yv + vi, q);
          }
        } else {
#pragma unroll
          for (int k = 0; k < PER; ++k) {
            const int j = k * T6S_THREADS + tid;
            if (j < n) Y[orow + t0 + j] = tile[j + (j >> 5)];
          }
        }
        run = tilesum;
        __syncthreads();
      }
      carry = Arith<V>::add(carry, segtot);
      buf ^= 1;
    }
  }
}

// ---- single-pass streaming scan (long unit-stride rows; the default) ---------------
// One CTA per SM, persistent.  The row is cut into segments of G·W elements; CTA b owns
// elements [b·W, (b+1)·W) of every segment.  Its slice is brought into shared memory by
// one TMA bulk copy (cp.async.bulk, mbarrier complete_tx) issued three jobs ahead into a
// ring of four buffers, so HBM reads stream while the current segment is scanned.
// Per segment: (A) thread sums of K consecutive elements (K odd: conflict-free banks) and
// the CTA total, published with a (launch epoch, job) tag in an 8-slot ring; (B) exclusive
// prefix = carry + Σ totals of lower CTAs (fixed order, polled by warp 0 — no grid barrier;
// the carry adds ALL totals of the previous segment, which keeps every CTA within two jobs
// of the slowest, so the ring never laps); (A) of the next job runs before (B), so the
// poll finds the other CTAs' totals already published; (C) in-place sequential scan of each
// thread's K elements from (prefix + its exclusive offset), proxy fence, one bulk store to
// the output.  HBM: one read + one write per element; deterministic (fixed association).
constexpr int T6T_THREADS = 256, T6T_NBUF = 4;   // EXPERIMENT: two CTAs per SM
template <class V> struct T6K { static constexpr int K = sizeof(V) == 4 ? 27 : 13; };
template <class V> constexpr int t6_w() { return T6T_THREADS * T6K<V>::K; }
template <class V> constexpr int t6_smem() { return T6T_NBUF * t6_w<V>() * (int)sizeof(V) + 128; }

__device__ __forceinline__ void t6_mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile("{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}"
               ::"r"(bar), "r"(parity) : "memory");
}

// CTA totals travel as self-validating 64-bit words (tag << 32 | 32 value bits; 8-byte
// values use two such words): one aligned 64-bit store publishes, one 64-bit load both
// checks and reads — single-copy atomic, so no fences and one L2 round trip per poll.
__device__ __forceinline__ unsigned t6_tag(unsigned epoch, long long job) {
  return epoch * 0x9E3779B1u + (unsigned)job + 1u;
}
template <class V>
__device__ __forceinline__ void t6_publish(unsigned long long* slot, unsigned tag, V v) {
  const unsigned long long t = (unsigned long long)tag << 32;
  if constexpr (sizeof(V) == 4) {
    *(volatile unsigned long long*)slot = t | __float_as_uint(*reinterpret_cast<const float*>(&v));
  } else {
    const unsigned long long u = *reinterpret_cast<const unsigned long long*>(&v);
    *(volatile unsigned long long*)slot = t | (u & 0xFFFFFFFFull);
    *(volatile unsigned long long*)(slot + 1) = t | (u >> 32);
  }
}
template <class V>
__device__ __forceinline__ bool t6_read(const unsigned long long* slot, unsigned tag, V* v) {
  if constexpr (sizeof(V) == 4) {
    const unsigned long long w = *(volatile const unsigned long long*)slot;
    const unsigned lo = (unsigned)w;
    *v = *reinterpret_cast<const V*>(&lo);
    return (unsigned)(w >> 32) == tag;
  } else {
    const unsigned long long w0 = *(volatile const unsigned long long*)slot;
    const unsigned long long w1 = *(volatile const unsigned long long*)(slot + 1);
    const unsigned long long u = (w0 & 0xFFFFFFFFull) | (w1 << 32);
    *v = *reinterpret_cast<const V*>(&u);
    return (unsigned)(w0 >> 32) == tag && (unsigned)(w1 >> 32) == tag;
  }
}

// Warp 0: (Σ_{i<G} prev[i], Σ_{i<b} cur[i]) once their tags match — lane-strided
// sequential sums, then a fixed shuffle tree (deterministic for a given G, b); all the
// reads of a lane are issued together (G ≤ 320: 10 per lane and slot)
template <class V>
__device__ __forceinline__ void t6_sums_tagged(const unsigned long long* pw, unsigned ptag, bool want_prev,
                                               const unsigned long long* cw, unsigned ctag, int G, int b,
                                               V* all_prev, V* lower) {
  constexpr int R = 10, S = sizeof(V) == 4 ? 1 : 2;
  const int lane = threadIdx.x;
  bool okp[R], okc[R];
  V vp[R], vc[R];
#pragma unroll
  for (int u = 0; u < R; ++u) {
    const int i = lane + 32 * u;
    okp[u] = !want_prev || i >= G;
    okc[u] = i >= b;
    vp[u] = (V)0;
    vc[u] = (V)0;
  }
  while (true) {
    bool done = true;
#pragma unroll
    for (int u = 0; u < R; ++u) {
      const int i = lane + 32 * u;
      if (!okp[u]) okp[u] = t6_read<V>(pw + S * i, ptag, &vp[u]);
      if (!okc[u]) okc[u] = t6_read<V>(cw + S * i, ctag, &vc[u]);
      done = done && okp[u] && okc[u];
    }
    if (__all_sync(0xffffffffu, done)) break;
    __nanosleep(20);
  }
  V a = (V)0, c = (V)0;
#pragma unroll
  for (int u = 0; u < R; ++u) {
    const int i = lane + 32 * u;
    if (want_prev && i < G) a = Arith<V>::add(a, vp[u]);
    if (i < b) c = Arith<V>::add(c, vc[u]);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    a = Arith<V>::add(a, __shfl_down_sync(0xffffffffu, a, o));
    c = Arith<V>::add(c, __shfl_down_sync(0xffffffffu, c, o));
  }
  *all_prev = __shfl_sync(0xffffffffu, a, 0);
  *lower = __shfl_sync(0xffffffffu, c, 0);
}

template <class V>
__global__ void __launch_bounds__(T6T_THREADS, 2) t6_stream_scan_kernel(const __grid_constant__ T6Params P) {
  constexpr int K = T6K<V>::K, W = t6_w<V>(), VEC = 16 / sizeof(V), NB = T6T_NBUF;
  extern __shared__ __align__(128) uint8_t t6_dyn[];
  V* buf = reinterpret_cast<V*>(t6_dyn);                            // [NB][W] (stays in the shared window)
  __shared__ __align__(8) uint64_t mbar[NB];
  __shared__ V red[2][T6T_THREADS / 32];
  __shared__ V s_pre;
  __shared__ unsigned s_epoch;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int G = gridDim.x, b = blockIdx.x;
  unsigned* hdr = (unsigned*)P.loc;
  // CTA totals (tagged words) in an 8-slot ring: a CTA at iteration i writes job i+1 while
  // the slowest CTA (≥ iteration i-2, see B) may still read jobs i-3 and i-2
  constexpr int SW = sizeof(V) == 4 ? 1 : 2;
  unsigned long long* part = (unsigned long long*)P.z;       // [8][G][SW]
  const V* X = (const V*)P.ptr[0];
  V* Y = (V*)P.out;
  const int64_t SEG = (int64_t)G * W;
  const int64_t nseg = (P.T + SEG - 1) / SEG, njobs = P.Nc * nseg;
  if (tid == 0) {
    s_epoch = *(volatile unsigned*)hdr + 1u;
    for (int i = 0; i < NB; ++i)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&mbar[i])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const unsigned E = s_epoch;
  // job j = (row, segment): input/output offsets of this CTA's slice [e, e + len)
  auto job = [&](int64_t j, int64_t* xo, int64_t* yo, int* len, int64_t* sg) {
    const int64_t c = j / nseg, sgi = j % nseg;
    int64_t xrow = P.base[0], rem = c;
    for (int d = P.nrowd - 1; d >= 0; --d) {
      const int64_t v = rem % P.rowsize[d];
      rem /= P.rowsize[d];
      xrow += P.Lrow[0][d] * v;
    }
    const int64_t e = sgi * SEG + (int64_t)b * W;
    *len = (int)max((int64_t)0, min((int64_t)W, P.T - e));
    *xo = xrow + e;
    *yo = t6_out_offset(P, c, 0) + e;
    *sg = sgi;
  };
  auto bulk_elems = [&](const void* base, int64_t off, int len) -> int {   // 16-B aligned, whole vectors
    return ((((uintptr_t)base + off * sizeof(V)) & 15) == 0) ? len / VEC * VEC : 0;
  };
  auto issue = [&](int64_t j) {        // thread 0: TMA bulk load of job j's slice into buffer j % NB
    int64_t xo, yo, sg;
    int len;
    job(j, &xo, &yo, &len, &sg);
    const int nb = bulk_elems(X, xo, len);
    const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&mbar[j % NB]);
    const uint32_t dst = (uint32_t)__cvta_generic_to_shared(buf + (j % NB) * W);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"((uint32_t)(nb * sizeof(V))) : "memory");
    if (nb > 0)
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(dst), "l"(X + xo), "r"((uint32_t)(nb * sizeof(V))), "r"(bar) : "memory");
  };
  // (A) of job j: wait for its slice, fill unaligned/tail elements, thread sums of K
  // consecutive elements (K odd: conflict-free banks), warp scan, CTA total published
  auto phaseA = [&](int64_t j, V* incl_out) {
    int64_t xo, yo, sg;
    int len;
    job(j, &xo, &yo, &len, &sg);
    V* sb = buf + (j % NB) * W;
    t6_mbar_wait((uint32_t)__cvta_generic_to_shared(&mbar[j % NB]), (uint32_t)((j / NB) & 1));
    const int nb = bulk_elems(X, xo, len);
    for (int i = nb + tid; i < len; i += T6T_THREADS) sb[i] = X[xo + i];
    __syncthreads();
    const int k0 = tid * K, k1 = min(len, k0 + K);
    V ts = (V)0;
    if (k1 - k0 == K) {            // whole run: all K shared-memory loads issued before the adds
      V v[K];
#pragma unroll
      for (int q = 0; q < K; ++q) v[q] = sb[k0 + q];
#pragma unroll
      for (int q = 0; q < K; ++q) ts = Arith<V>::add(ts, v[q]);
    } else {
      for (int k = k0; k < k1; ++k) ts = Arith<V>::add(ts, sb[k]);
    }
    V incl = ts;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const V nbv = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl = Arith<V>::add(nbv, incl);
    }
    V* rd = red[j & 1];
    if (lane == 31) rd[warp] = incl;
    __syncthreads();
    if (tid == 0) {
      V tot = rd[0];
      for (int w = 1; w < T6T_THREADS / 32; ++w) tot = Arith<V>::add(tot, rd[w]);
      t6_publish<V>(part + ((j & 7) * G + b) * SW, t6_tag(E, j), tot);
    }
    *incl_out = incl;
  };
  if (tid == 0)
    for (int64_t j = 0; j < NB - 1 && j < njobs; ++j) issue(j);
  V carry = (V)0, incl_cur = (V)0;
  if (njobs > 0) phaseA(0, &incl_cur);
  for (int64_t j = 0; j < njobs; ++j) {
    int64_t xo, yo, sg;
    int len;
    job(j, &xo, &yo, &len, &sg);
    V* sb = buf + (j % NB) * W;
    // next job's (A) first: its wait overlaps the other CTAs publishing job j
    V incl_next = (V)0;
    if (j + 1 < njobs) phaseA(j + 1, &incl_next);
    // (B) carry over the previous segment (all CTAs), prefix of the lower CTAs of job j
    if (warp == 0) {
      const int ps = (int)((j + 7) & 7), cs = (int)(j & 7);
      V all, lower;
      t6_sums_tagged<V>(part + ps * G * SW, t6_tag(E, j - 1), j > 0, part + cs * G * SW, t6_tag(E, j), G, b, &all,
                        &lower);
      if (j > 0) carry = sg == 0 ? (V)0 : Arith<V>::add(carry, all);
      if (lane == 0) s_pre = Arith<V>::add(carry, lower);
    }
    __syncthreads();
    // (C) in-place scan of job j from (prefix + this thread's exclusive offset), bulk store
    const V* rd = red[j & 1];
    V base = s_pre;
    for (int w = 0; w < warp; ++w) base = Arith<V>::add(base, rd[w]);
    const V prev = __shfl_up_sync(0xffffffffu, incl_cur, 1);
    V r = lane == 0 ? base : Arith<V>::add(base, prev);
    const int k0 = tid * K, k1 = min(len, k0 + K);
    if (k1 - k0 == K) {            // whole run: loads first, then the sequential scan and stores
      V v[K];
#pragma unroll
      for (int q = 0; q < K; ++q) v[q] = sb[k0 + q];
#pragma unroll
      for (int q = 0; q < K; ++q) {
        r = Arith<V>::add(r, v[q]);
        sb[k0 + q] = r;
      }
    } else {
      for (int k = k0; k < k1; ++k) {
        r = Arith<V>::add(r, sb[k]);
        sb[k] = r;
      }
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    const int ob = bulk_elems(Y, yo, len);
    for (int i = ob + tid; i < len; i += T6T_THREADS) Y[yo + i] = sb[i];
    if (tid == 0) {
      if (ob > 0) {
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                     ::"l"(Y + yo), "r"((uint32_t)__cvta_generic_to_shared(sb)), "r"((uint32_t)(ob * sizeof(V))) : "memory");
      }
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      // refill the buffer of job j-1 with job j+3 once its store has read it (one group may
      // stay in flight: job j's store); job j+3 is consumed two iterations later
      if (j + NB - 1 < njobs) {
        asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        issue(j + NB - 1);
      }
    }
    // (no barrier here: red[j & 1] is next written after phaseA's first barrier, s_pre after
    // its second, and this job's buffer is refilled only after the next iteration's barriers)
    incl_cur = incl_next;
  }
  if (tid == 0) {
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    // the last CTA out advances the epoch
    __threadfence();
    if (atomicAdd(hdr + 1, 1u) == (unsigned)G - 1) {
      hdr[1] = 0u;
      __threadfence();
      atomicAdd(hdr, 1u);
    }
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
  const int dps = p->ps[0];
  const int64_t T = p->size[dps];
  const int64_t Nc = p->Ncc / T;
  const int64_t nq = (T + T6_CHUNK - 1) / T6_CHUNK;
  const int64_t vs = vsize(p->compute);
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  // single-pass segmented scan: input read directly (no pw dims, identity), unit strides
  // along the ps dim, input/output already in the compute type, rows of ≥ 64 Ki elements
  const bool seg = p->nred == 1 && p->f == MDH_F_IDENTITY && p->n_in_acc == 1 && p->in[0].dtype == p->compute &&
                   p->out[0].dtype == p->compute && p->in[0].acc[0].L[dps] == 1 && p->out[0].acc[0].L[dps] == 1 &&
                   T >= 65536 && p->tiles.seg >= 0;
  if (seg && p->tiles.seg > 0) {          // segmented variant (tile knob seg = elements per segment)
    int64_t sl = std::max<int64_t>(T6S_UNIT, (int64_t)p->tiles.seg / T6S_UNIT * T6S_UNIT);
    p->auxi.assign(1, sl);
    p->tiles.seg = (int)std::min<int64_t>(sl, INT32_MAX);
    p->ws_kernel = 256 + al((size_t)2 * 148 * 8 * vs);
    return MDH_OK;
  }
  if (seg) {                              // streaming scan (default)
    p->auxi.assign(1, -1);
    p->ws_kernel = 256 + al((size_t)8 * 320 * 16);     // header, 8 × G tagged totals
    return MDH_OK;
  }
  p->auxi.clear();
  p->ws_kernel = al((size_t)Nc * T * vs) + (nq > 1 ? al((size_t)Nc * T * vs) + al((size_t)Nc * nq * vs) : 0);
  // column fold (t6_colfold_kernel): fp32, one pw dim, the ps dim unit-stride, few points
  // (≤ 2^20) — room for T6_COL_SMAX split partials and the per-group tickets
  int npw = 0;                            // pw dims (p->red also lists the ps dim)
  for (int t = 0; t < p->nred; ++t) npw += p->red[t] != dps;
  const bool col = npw == 1 && p->f == MDH_F_IDENTITY && p->n_in_acc == 1 && p->in[0].dtype == MDH_F32 &&
                   p->compute == MDH_F32 && p->in[0].acc[0].L[dps] == 1 && T % 4 == 0 && Nc * T <= (1 << 20);
  if (col) {
    p->auxi.assign(2, 0);
    p->auxi[0] = -2;                      // marker: column fold eligible (launch re-checks alignment)
    p->auxi[1] = (int64_t)p->ws_kernel;   // offset of the split partials
    p->ws_kernel += al((size_t)T6_COL_SMAX * Nc * T * 4) + al((size_t)Nc * ((T + 127) / 128) * 4);
  }
  return MDH_OK;
}

template <class V>
static mdh_status launch_seg(const T6Params& P0, char* ws, cudaStream_t st) {
  T6Params P = P0;
  static int o = 0;                      // resident CTAs per SM (cached per instantiation)
  if (o == 0) {
    MDH_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, t6_seg_scan_kernel<V>, T6S_THREADS, 0));
    o = std::max(1, std::min(o, 8));
  }
  int dev = 0, sms = 148;
  MDH_CUDA(cudaGetDevice(&dev));
  MDH_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  const int G = std::min(sms * o, 148 * 8);
  P.loc = ws;                            // grid-barrier counters (zero at rest)
  P.sums = ws + 256;                     // CTA totals [2][G]
  void* args[] = {&P};
  MDH_CUDA(cudaLaunchCooperativeKernel((const void*)t6_seg_scan_kernel<V>, dim3(G), dim3(T6S_THREADS), args, 0, st));
  return post_launch("t6_seg_scan_kernel");
}

template <class V>
static mdh_status launch_stream(T6Params& P, cudaStream_t st) {
  // one attribute call per instantiation (a function-local static of the template: V = 4-
  // and 8-byte types each get their own; indexing a shared array by sizeof(V) overran it)
  static std::once_flag once;
  static cudaError_t aerr = cudaSuccess;
  std::call_once(once, [] {
    aerr = cudaFuncSetAttribute((const void*)t6_stream_scan_kernel<V>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                t6_smem<V>());
  });
  MDH_CUDA(aerr);
  int dev = 0, sms = 148;
  MDH_CUDA(cudaGetDevice(&dev));
  MDH_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  static int per = 0;                     // resident CTAs per SM (2 for every value type)
  if (per == 0) {
    MDH_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, t6_stream_scan_kernel<V>, T6T_THREADS, t6_smem<V>()));
    per = std::max(1, std::min(per, 2));
  }
  const int G = std::min(per * sms, 320);  // co-resident (cooperative launch); ≤ 320: 10 tags per polling lane
  void* args[] = {&P};
  MDH_CUDA(cudaLaunchCooperativeKernel((const void*)t6_stream_scan_kernel<V>, dim3(G), dim3(T6T_THREADS), args,
                                       t6_smem<V>(), st));
  return post_launch("t6_stream_scan_kernel");
}

// every output row starts on a 16-byte boundary (float4 stores in t6_rowscan4_kernel)
static bool row_out_aligned4(const T6Params& P) {
  if (((uintptr_t)P.out & 15) != 0 || ((uintptr_t)P.z & 15) != 0 || P.obase % 4 != 0) return false;
  for (int q = 0; q < P.nrowd; ++q)
    if (P.orowL[q] % 4 != 0) return false;
  return true;
}

template <class V>
static mdh_status launch_typed(const T6Params& P, cudaStream_t st) {
  const int64_t total = P.Nc * P.T;
  const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>((total + 255) / 256, 148LL * 32));
  if (!P.direct) {
    // sub-ranges per point: 32 when the pw range is long and the points alone cannot fill
    // the GPU (MBBS: 8192 points × 8192 rows), else 8
    int64_t npts = 1;
    for (int q = 0; q < P.npw; ++q) npts *= P.pwsize[q];
    if (std::is_same<V, float>::value && P.colS > 0) {
      const unsigned groups = (unsigned)(P.Nc * ((P.T + 127) / 128));
      t6_colfold_kernel<<<dim3(groups, (unsigned)P.colS), dim3(32, 8), 0, st>>>(P);
      MDH_TRY(post_launch("t6_colfold_kernel"));
    } else {
      const int Y = (npts >= 1024 && total < 148LL * 2048) ? 32 : 8;
      const unsigned gf = (unsigned)std::max<int64_t>(1, std::min<int64_t>((total + 31) / 32, 148LL * 64));
      t6_fold_kernel<V><<<gf, dim3(32, Y), 0, st>>>(P);
      MDH_TRY(post_launch("t6_fold_kernel"));
    }
  }
  if (std::is_same<V, float>::value && !P.direct && P.colS > 0 && P.odt == MDH_F32 && P.oLt == 1 &&
      P.T % 4096 == 0 && P.T <= 8 * 4096 && P.Nc <= INT32_MAX && row_out_aligned4(P)) {
    // fp32 rows after the column fold: register row scan, launched as a programmatic
    // dependent of the fold (its launch and prologue overlap the fold's tail)
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)P.Nc);
    cfg.blockDim = dim3(1024);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    MDH_CUDA(cudaLaunchKernelEx(&cfg, t6_rowscan4_kernel, P));
    return post_launch("t6_rowscan4_kernel");
  }
  if (!P.direct && P.T * (int64_t)sizeof(V) <= T6_ROW_SMEM && P.Nc <= INT32_MAX) {
    // short rows: one single-block scan per row instead of chunk scan + totals + fix-up
    t6_rowscan_kernel<V><<<(unsigned)P.Nc, 1024, (size_t)P.T * sizeof(V), st>>>(P);
    return post_launch("t6_rowscan_kernel");
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
  if (p.auxi.size() == 1 && p.auxi[0] == -1) {    // streaming scan (prepare_t6)
    P.loc = w;                                      // header: epoch, done counter
    P.z = w + 256;                                  // tagged CTA totals [8][G]
    switch (p.compute) {
      case MDH_F32: return launch_stream<float>(P, st);
      case MDH_F64: return launch_stream<double>(P, st);
      case MDH_I32: return launch_stream<int32_t>(P, st);
      case MDH_U32: return launch_stream<uint32_t>(P, st);
      case MDH_I64: return launch_stream<long long>(P, st);
      default: set_error("T6: unsupported type"); return MDH_ERR_UNSUPPORTED;
    }
  }
  const bool colfold = p.auxi.size() == 2 && p.auxi[0] == -2;
  if (!p.auxi.empty() && !colfold) {      // segmented single-pass scan (prepare_t6)
    P.nq = p.auxi[0];
    switch (p.compute) {
      case MDH_F32: return launch_seg<float>(P, w, st);
      case MDH_F64: return launch_seg<double>(P, w, st);
      case MDH_I32: return launch_seg<int32_t>(P, w, st);
      case MDH_U32: return launch_seg<uint32_t>(P, w, st);
      case MDH_I64: return launch_seg<long long>(P, w, st);
      default: set_error("T6: unsupported type"); return MDH_ERR_UNSUPPORTED;
    }
  }
  P.z = w;
  P.loc = w + al((size_t)P.Nc * P.T * vs);
  P.sums = (char*)P.loc + al((size_t)P.Nc * P.T * vs);
  if (colfold && !P.direct) {
    // 16-byte loads need every point's first element 16-byte aligned
    bool aligned = (uintptr_t)P.ptr[0] % 16 == 0 && P.base[0] % 4 == 0;
    for (int q = 0; q < P.nrowd; ++q) aligned &= P.Lrow[0][q] % 4 == 0;
    aligned &= P.Lpw[0][0] % 4 == 0;
    if (aligned) {
      int dev = 0, sms = 148;
      MDH_CUDA(cudaGetDevice(&dev));
      MDH_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
      const int64_t groups = P.Nc * ((P.T + 127) / 128);
      // splits so that the blocks fill 8 × 256 threads per SM, rows per thread ≥ 32
      int64_t S = std::max<int64_t>(1, (int64_t)sms * 8 / std::max<int64_t>(1, groups));
      S = std::min<int64_t>({S, (int64_t)T6_COL_SMAX, std::max<int64_t>(1, P.pwsize[0] / 256)});
      if (p.tiles.split > 0) S = std::min<int64_t>({(int64_t)p.tiles.split, (int64_t)T6_COL_SMAX, P.pwsize[0]});   // tile knob
      P.colS = (int)S;
      P.colpart = (float*)(w + p.auxi[1]);
      P.colcnt = (unsigned*)(w + p.auxi[1] + al((size_t)T6_COL_SMAX * P.Nc * P.T * 4));
    }
  }
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
