// internal.h — shared definitions of libmdh (planner, kernels, ABI).
//
// The plan turns the paper's problem statement (md_hom + inp_view/out_view, Listing 7
// P:223-251) into the linearised form every kernel works on:
//
//   element offset of access a at point i  =  base_a + Σ_d L_a[d] · i_d
//
// where L_a[d] = Σ_r coeff[r][d]·rowstride[r] and base_a = Σ_r offset[r]·rowstride[r]
// (row-major buffers, Listing 1 `M[i*K+k]` P:91; affine index functions, reading C-8).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <mutex>
#include <string>
#include <vector>

#include "../../include/mdh.h"

namespace mdh {

enum Template : int {
  T0_GENERIC = 0,   // any valid spec: one thread per cc point, literal fold (catch-all)
  T1_STENCIL = 1,   // all-cc shift stencil / map (Jacobi1D/3D)
  T2_REDUCE = 2,    // streaming reduction (Dot, MatVec, row/column reductions)
  T3_SIMT = 3,      // fp32/int32 SIMT contraction (MatMul fp32, CCSD(T)/MCC fp32)
  T4_TC = 4,        // bf16 tcgen05 contraction (MatMul, CCSD(T), MCC)
  T5_PRL = 5,       // pairwise record linkage with custom ordered combine
  T6_SCAN = 6       // ps(add) prefix sums (Listing 17; MBBS)
};

const char* template_name(int t);

struct Access {
  int64_t base;
  int64_t L[MDH_MAX_D];
};

struct Buf {
  mdh_dtype dtype;
  int rank;
  int64_t shape[MDH_MAX_RANK];       // local (this rank's) shape
  int64_t gshape[MDH_MAX_RANK];      // global shape
  int64_t goff[MDH_MAX_RANK];        // global coordinate of local element 0
  int64_t elems;
  int nacc;
  Access acc[MDH_MAX_ACC];
  mdh_index_fn fn[MDH_MAX_ACC];      // local index functions (after shard rewrite)
};

// Contraction grouping (T3/T4): dims split into batch (Z), M (A only), N (B only), K (pw).
struct Contraction {
  int nz = 0, nm = 0, nn = 0, nk = 0;
  int zd[MDH_MAX_D], md[MDH_MAX_D], nd[MDH_MAX_D], kd[MDH_MAX_D];
  int64_t Z = 1, M = 1, N = 1, K = 1;
  int a_buf = 0, b_buf = 1;          // which input plays A (uses M) and B (uses N)
};

struct Tiles {
  // generic knobs, interpreted per template (see tiles.cpp / tiles/b200.json)
  int threads = 256;
  int bm = 128, bn = 128, bk = 8;
  int split = 0;                      // 0 = auto
  int stages = 4;
  int vec = 4;
  int zchunk = 32;
  int seg = 0;                        // T6: elements per L2-resident scan segment (0 = auto)
  int per_thread = 1;
  int cluster = 1;
  int implicit = 0;                   // T4 A operand when not 2-D: 0 auto, 1 N-d TMA box (implicit
                                      // GEMM), 2 in-kernel cp.async gather, 3 gather pre-pass
  int epi = 0;                        // T4 scatter epilogue: 0 auto, 1 never the bulk-run (EPI 3) kernel
  int krot = 0;                       // T4 k-block rotation per tile (1 = on)
  int l2pf = 0;                       // T1 7-point row loads: L2 prefetch hint 0 none, 1 128 B, 2 256 B
  int areuse = -1;                    // T4 2-SM wide: k-outer MMA order reusing A from the collector (-1 auto = on, 0 off)
  int nstream = -1;                   // T4 2-SM wide: column-unit stream schedule (-1 auto, 0 off, 1 on)
  int mode = -1;                      // T1 7-point: -1 auto, 0 per-thread rows, 1 warp-coalesced rows,
                                      // 2 warp-coalesced + y-neighbour rows shared through smem
  std::string source = "default";
};

struct Plan {
  // ---- spec (local after shard rewrite) ----
  int D = 0;
  int64_t size[MDH_MAX_D] = {0};
  mdh_combine op[MDH_MAX_D];
  mdh_fn f = MDH_F_MUL;
  std::vector<double> fparams;
  int n_in = 0, n_out = 0;
  Buf in[MDH_MAX_BUFS];
  Buf out[MDH_MAX_BUFS];
  int n_in_acc = 0;                   // total input accesses
  // ---- classification ----
  int ncc = 0, nred = 0, nps = 0;
  int cc[MDH_MAX_D], red[MDH_MAX_D];  // cc: kept dims (cc and ps); red: folded dims (pw and ps)
  int ps[MDH_MAX_D];                  // prefix-sum dims (Listing 17)
  mdh_combine redop = MDH_CC;         // the common pw operator (reading C-3), CC if none
  int64_t Ncc = 1, Nred = 1;
  mdh_dtype compute = MDH_F32;        // arithmetic type of f and ⊕
  int tmpl = T0_GENERIC;
  Contraction con;
  Tiles tiles;
  std::string why;                    // reason for the template choice
  // ---- multi-GPU ----
  int device = 0, world = 1, rank = 0, shard_dim = -1;
  uint32_t flags = 0;
  void* comm = nullptr;
  bool sharded = false;               // the shard rewrite ran (world > 1, or a one-rank NCCL shard)
  bool shard_is_red = false;
  int64_t shard_start = 0, shard_len = 0, global_size = 0;
  // ---- workspace ----
  size_t ws_kernel = 0;               // bytes the template needs
  size_t ws_comm = 0;                 // bytes for gathered partials (pw shard)
  size_t ws_total = 0;
  // ---- plan-owned device constants: built on the host at plan time (no GPU needed),
  // uploaded once on the first execute (lazily, under a mutex), freed by mdh_destroy ----
  std::vector<uint8_t> host_const;
  size_t tab_off[16] = {0};           // byte offsets of the individual tables
  mutable void* dconst = nullptr;
  mutable std::mutex mu;
  void* tmaps = nullptr;              // T4: host copy of CUtensorMap descriptors
  int t4_variant = 0;
  std::vector<int64_t> auxi;          // template-specific host data (e.g. T1 stencil shape)
  std::vector<double> auxd;
};

// device pointer of the plan's constants (uploads them on first use)
mdh_status device_consts(const Plan& p, const char** base);
// append a table to host_const (256-byte aligned); returns its byte offset
size_t add_const(Plan* p, const void* data, size_t bytes);

// -------------------------------------------------------------------- errors
void set_error(const char* fmt, ...);
#define MDH_TRY(x)                               \
  do {                                           \
    mdh_status _s = (x);                         \
    if (_s != MDH_OK) return _s;                 \
  } while (0)
mdh_status cuda_check(cudaError_t e, const char* what);
#define MDH_CUDA(x) MDH_TRY(::mdh::cuda_check((x), #x))

int64_t dtype_size(mdh_dtype t);
bool is_float(mdh_dtype t);

// launch counter (per thread), reported by mdh_last_launch_count
void count_launch(int n = 1);
void reset_launch_count();
int launch_count();
mdh_status post_launch(const char* what);

// ---------------------------------------------------------------- planner
mdh_status build_plan(const mdh_spec* spec, const mdh_plan_opts* opts, Plan* p);
std::string describe_plan(const Plan& p);
void lookup_tiles(Plan* p, const char* table_path, const char* force);

// ---------------------------------------------------------------- templates
// Each launcher enqueues on `st`; `ws` is the kernel part of the workspace.
mdh_status prepare_t0(Plan* p);
mdh_status launch_t0(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st);
mdh_status prepare_t1(Plan* p);
mdh_status launch_t1(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st);
mdh_status launch_t1_halo(const Plan& p, const void* in, void* out, void* hlo, void* hhi, cudaStream_t st,
                          bool pdl = false);
mdh_status prepare_t2(Plan* p);
mdh_status launch_t2(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st);
mdh_status prepare_t3(Plan* p);
mdh_status launch_t3(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st);
mdh_status prepare_t4(Plan* p);
mdh_status launch_t4(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st);
bool t4_supported(const Plan& p, std::string* why);
// T4 small-K direct contraction (t4_conv.cu): true if the plan was set up for it
bool prepare_t4_conv(Plan* p);
mdh_status launch_t4_conv(const Plan& p, const void* const* in, void* const* out, cudaStream_t st);
mdh_status prepare_t5(Plan* p);
mdh_status launch_t5(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st);
mdh_status prepare_t6(Plan* p);
mdh_status launch_t6(const Plan& p, const void* const* in, void* const* out, void* ws, cudaStream_t st);
void release_t4(Plan* p);

// measured instruction-throughput peaks (peaks.cu; diagnostics)
mdh_status measure_peaks(int device, double* ffma_tflops, double* alu_tops, double* issue_tops);

// ordered ⊗-fold of S partial output sets (K-combine)
mdh_status launch_combine(const Plan& p, const void* const* partials, int S, void* const* out,
                          cudaStream_t st);

// ---------------------------------------------------------------- comm (NCCL via dlopen)
mdh_status comm_unique_id(void* id128);
mdh_status comm_init(const void* id128, int world, int rank, int device, void** comm);
mdh_status comm_destroy(void* comm);
mdh_status comm_allgather(void* comm, const void* send, void* recv, size_t bytes, cudaStream_t st);
mdh_status comm_halo_exchange(void* comm, int rank, int world, char* buf, size_t plane_bytes, int64_t nz,
                              cudaStream_t st);
mdh_status comm_allreduce(void* comm, const void* send, void* recv, size_t count, mdh_dtype dt,
                          mdh_combine op, cudaStream_t st);

}  // namespace mdh
