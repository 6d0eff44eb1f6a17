// abi.cpp — the extern "C" entry points of libmdh (include/mdh.h).
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>

#include "internal.h"

#include <mutex>
#include <vector>

// Pipelined host execution (mdh_execute_host): the problem cut into C chunks along a cc
// dim on which every buffer depends only through its outermost coordinate, so each chunk's
// input and output slices are contiguous host ranges.  Chunk c's H2D copies (copy-in
// stream), its computation (the caller's stream; sub-plan = virtual shard c of C) and its
// D2H copies (copy-out stream) overlap the neighbouring chunks' — both PCIe directions and
// the GPU busy at once.
struct HostPipe {
  bool built = false, ok = false;
  int dim = -1, C = 0;
  std::vector<mdh_plan_t> sub;
  size_t ws_max = 0;
  cudaStream_t s_in = nullptr, s_out = nullptr;
  std::vector<cudaEvent_t> ev;        // [0] entry, [1..C] copied in, [C+1..2C] computed, [2C+1] copied out
};

struct mdh_plan_s {
  mdh::Plan p;
  // a copy of the spec and options (world_size 1 plans): the pipeline's sub-plans
  bool have_spec = false;
  mdh_spec spec{};
  std::vector<mdh_buffer> sin, sout;
  std::vector<double> fpar;
  mdh_plan_opts opts{};
  std::string tile_table, force_tile;
  std::mutex mu;
  HostPipe pipe;
};

namespace mdh {

static thread_local std::string g_err;
static thread_local int g_launches = 0;

void set_error(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  std::vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
}

mdh_status cuda_check(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return MDH_OK;
  set_error("CUDA error in %s: %s", what, cudaGetErrorString(e));
  return e == cudaErrorMemoryAllocation ? MDH_ERR_OUT_OF_MEMORY : MDH_ERR_CUDA;
}

int64_t dtype_size(mdh_dtype t) {
  switch (t) {
    case MDH_BF16: return 2;
    case MDH_F32: case MDH_I32: case MDH_U32: return 4;
    case MDH_F64: case MDH_I64: return 8;
  }
  return 0;
}

bool is_float(mdh_dtype t) { return t == MDH_BF16 || t == MDH_F32 || t == MDH_F64; }

void count_launch(int n) { g_launches += n; }
void reset_launch_count() { g_launches = 0; }
int launch_count() { return g_launches; }

static bool debug_sync() {
  static int v = -1;
  if (v < 0) {
    const char* e = std::getenv("MDH_DEBUG_SYNC");
    v = (e && e[0] == '1') ? 1 : 0;
  }
  return v == 1;
}

mdh_status post_launch(const char* what) {
  count_launch(1);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_check(e, what);
  if (debug_sync()) return cuda_check(cudaDeviceSynchronize(), what);
  return MDH_OK;
}

size_t add_const(Plan* p, const void* data, size_t bytes) {
  size_t off = (p->host_const.size() + 255) / 256 * 256;
  p->host_const.resize(off + bytes);
  std::memcpy(p->host_const.data() + off, data, bytes);
  return off;
}

mdh_status device_consts(const Plan& p, const char** base) {
  std::lock_guard<std::mutex> g(p.mu);
  if (!p.dconst && !p.host_const.empty()) {
    void* d = nullptr;
    MDH_CUDA(cudaMalloc(&d, p.host_const.size()));
    cudaError_t e = cudaMemcpy(d, p.host_const.data(), p.host_const.size(), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
      cudaFree(d);
      return cuda_check(e, "upload of plan constants");
    }
    p.dconst = d;
  }
  *base = (const char*)p.dconst;
  return MDH_OK;
}

static mdh_status check_ptrs(const mdh::Plan& p, const void* const* in, void* const* out) {
  if (!in || !out) { set_error("in/out arrays are NULL"); return MDH_ERR_INVALID_ARG; }
  for (int b = 0; b < p.n_in; ++b) {
    if (!in[b]) { set_error("input %d is NULL", b); return MDH_ERR_INVALID_ARG; }
    if (reinterpret_cast<uintptr_t>(in[b]) % 16) { set_error("input %d is not 16-byte aligned", b); return MDH_ERR_INVALID_ARG; }
  }
  for (int b = 0; b < p.n_out; ++b) {
    if (!out[b]) { set_error("output %d is NULL", b); return MDH_ERR_INVALID_ARG; }
    if (reinterpret_cast<uintptr_t>(out[b]) % 16) { set_error("output %d is not 16-byte aligned", b); return MDH_ERR_INVALID_ARG; }
  }
  // aliasing (reading C-27)
  for (int b = 0; b < p.n_out; ++b) {
    uintptr_t o0 = (uintptr_t)out[b], o1 = o0 + (uintptr_t)(p.out[b].elems * dtype_size(p.out[b].dtype));
    for (int c = 0; c < p.n_in; ++c) {
      uintptr_t i0 = (uintptr_t)in[c], i1 = i0 + (uintptr_t)(p.in[c].elems * dtype_size(p.in[c].dtype));
      if (o0 < i1 && i0 < o1) { set_error("output %d overlaps input %d (reading C-27)", b, c); return MDH_ERR_INVALID_ARG; }
    }
  }
  return MDH_OK;
}

static mdh_status run_template(const mdh::Plan& p, const void* const* in, void* const* out, void* ws,
                               cudaStream_t st) {
  switch (p.tmpl) {
    case T0_GENERIC: return launch_t0(p, in, out, ws, st);
    case T1_STENCIL: return launch_t1(p, in, out, ws, st);
    case T2_REDUCE: return launch_t2(p, in, out, ws, st);
    case T3_SIMT: return launch_t3(p, in, out, ws, st);
    case T4_TC: return launch_t4(p, in, out, ws, st);
    case T5_PRL: return launch_t5(p, in, out, ws, st);
    case T6_SCAN: return launch_t6(p, in, out, ws, st);
  }
  set_error("unknown template");
  return MDH_ERR_INTERNAL;
}

// pw shard across ranks: local partial → allgather → ordered combine (ranks = index
// order), or an NCCL allreduce where ⊕ is exact in any order (int +, max, min).
static mdh_status execute_sharded(const mdh::Plan& p, const void* const* in, void* const* out, char* ws,
                                  cudaStream_t st) {
  size_t per = 0;
  size_t offs[MDH_MAX_BUFS];
  for (int b = 0; b < p.n_out; ++b) {
    offs[b] = per;
    per += ((size_t)p.out[b].elems * dtype_size(p.out[b].dtype) + 255) / 256 * 256;
  }
  char* local = ws + p.ws_kernel;                 // this rank's partial
  char* gathered = local + per;                   // world × per
  void* lout[MDH_MAX_BUFS];
  for (int b = 0; b < p.n_out; ++b) lout[b] = local + offs[b];
  MDH_TRY(run_template(p, in, lout, ws, st));
  bool exact_any_order = p.n_out == 1 && p.f != MDH_F_PRL_COMPARE &&
                         (p.redop == MDH_PW_MAX || p.redop == MDH_PW_MIN ||
                          (p.redop == MDH_PW_ADD && !is_float(p.out[0].dtype)));
  // opt-in: float sums through NCCL's reduction (order chosen by NCCL)
  const bool float_allreduce = (p.flags & MDH_PLAN_FLOAT_ALLREDUCE) && p.n_out == 1 && p.f != MDH_F_PRL_COMPARE &&
                               p.redop == MDH_PW_ADD && (p.out[0].dtype == MDH_F32 || p.out[0].dtype == MDH_F64);
  if (exact_any_order || float_allreduce) {
    // the reduction runs over the whole output buffer; elements outside the output image
    // must stay untouched (reading C-5), so reduce straight into out[0] only when the
    // (injective) image covers it, else in place in the workspace and place the image
    // with the S = 1 combine
    const bool covers = p.out[0].nacc == 1 && p.Ncc == p.out[0].elems;
    if (covers)
      return comm_allreduce(p.comm, lout[0], out[0], (size_t)p.out[0].elems, p.out[0].dtype, p.redop, st);
    MDH_TRY(comm_allreduce(p.comm, lout[0], lout[0], (size_t)p.out[0].elems, p.out[0].dtype, p.redop, st));
    const void* one[1] = {lout[0]};
    return launch_combine(p, one, 1, out, st);
  }
  MDH_TRY(comm_allgather(p.comm, local, gathered, per, st));
  const void* parts[MDH_MAX_WORLD * MDH_MAX_BUFS];
  for (int r = 0; r < p.world; ++r)
    for (int b = 0; b < p.n_out; ++b) parts[r * p.n_out + b] = gathered + (size_t)r * per + offs[b];
  return launch_combine(p, parts, p.world, out, st);
}

}  // namespace mdh

// Build the pipeline of a world-size-1 plan once (under h->mu): the first cc dim d on which
// every input and output buffer depends only through its coordinate 0 (or not at all),
// every output depending on it; C = 4 chunks as virtual shards of the plan on d.  Not
// built (ok = false) for small problems (< 32 MB of host data), when no dim qualifies, or
// with MDH_HOST_PIPE=0.
static void build_pipe(mdh_plan_s* h) {
  HostPipe& P = h->pipe;
  P.built = true;
  const mdh::Plan& p = h->p;
  if (!h->have_spec || p.world > 1 || p.sharded) return;
  const char* env = std::getenv("MDH_HOST_PIPE");
  if (env && env[0] == '0') return;
  size_t bytes = 0;
  for (int b = 0; b < p.n_in; ++b) bytes += (size_t)p.in[b].elems * mdh::dtype_size(p.in[b].dtype);
  for (int b = 0; b < p.n_out; ++b) bytes += (size_t)p.out[b].elems * mdh::dtype_size(p.out[b].dtype);
  const char* mn = std::getenv("MDH_HOST_PIPE_MIN_MB");      // (tests: pipeline small problems)
  if (bytes < ((size_t)(mn ? std::atoi(mn) : 32) << 20)) return;
  const mdh_spec& sp = h->spec;
  for (int d = 0; d < sp.D && !P.ok; ++d) {
    if (sp.op[d] != MDH_CC || sp.size[d] < 4) continue;
    bool ok = true;
    auto dep = [&](const mdh_buffer& B, bool* any) {
      *any = false;
      for (int a = 0; a < B.n_acc; ++a)
        for (int r = 0; r < B.rank; ++r)
          if (B.acc[a].coeff[r][d] != 0) {
            if (r != 0) ok = false;
            *any = true;
          }
    };
    bool any;
    for (int b = 0; b < sp.n_in; ++b) dep(sp.in[b], &any);
    for (int b = 0; b < sp.n_out; ++b) {
      dep(sp.out[b], &any);
      ok = ok && any;
    }
    if (!ok) continue;
    const char* ce = std::getenv("MDH_HOST_PIPE_CHUNKS");
    const int C = (int)std::min<int64_t>(ce ? std::max(2, std::atoi(ce)) : 4, sp.size[d]);
    std::vector<mdh_plan_t> sub(C, nullptr);
    size_t wsm = p.ws_total;
    for (int c = 0; c < C && ok; ++c) {
      mdh_plan_opts o = h->opts;
      o.world_size = C;
      o.rank = c;
      o.shard_dim = d;
      o.nccl_comm = nullptr;
      o.flags |= MDH_PLAN_VIRTUAL_SHARD;
      if (mdh_plan(&sp, &o, &sub[c]) != MDH_OK) {
        ok = false;
        break;
      }
      const mdh::Plan& q = sub[c]->p;
      wsm = std::max(wsm, q.ws_total);
      // slices must be contiguous: only coordinate 0 cut
      auto contiguous = [&](const mdh::Buf& L, const mdh::Buf& F) {
        for (int r = 1; r < F.rank; ++r)
          if (L.goff[r] != 0 || L.shape[r] != F.shape[r]) return false;
        return true;
      };
      for (int b = 0; b < p.n_in && ok; ++b) ok = contiguous(q.in[b], p.in[b]);
      for (int b = 0; b < p.n_out && ok; ++b) ok = contiguous(q.out[b], p.out[b]);
    }
    if (ok) {                           // the copy streams and events live on the plan's device
      int cur = 0;
      cudaGetDevice(&cur);
      cudaSetDevice(p.device);
      ok = cudaStreamCreateWithFlags(&P.s_in, cudaStreamNonBlocking) == cudaSuccess &&
           cudaStreamCreateWithFlags(&P.s_out, cudaStreamNonBlocking) == cudaSuccess;
      P.ev.assign(2 * C + 2, nullptr);
      for (auto& e : P.ev) ok = ok && cudaEventCreateWithFlags(&e, cudaEventDisableTiming) == cudaSuccess;
      cudaSetDevice(cur);
    }
    if (!ok) {
      for (auto q : sub) mdh_destroy(q);
      cudaGetLastError();
      continue;
    }
    P.ok = true;
    P.dim = d;
    P.C = C;
    P.sub = sub;
    P.ws_max = wsm;
  }
}

static void ensure_pipe(mdh_plan_s* h) {
  std::lock_guard<std::mutex> g(h->mu);
  if (!h->pipe.built) build_pipe(h);
}

static size_t host_bytes(const mdh::Buf& B) { return (size_t)B.elems * mdh::dtype_size(B.dtype); }

// elements of buffer F (full shape) before the slice L (coordinate 0 from goff[0]) and in it
static void slice_of(const mdh::Buf& L, const mdh::Buf& F, size_t* off, size_t* n) {
  size_t row = 1;
  for (int r = 1; r < F.rank; ++r) row *= (size_t)F.shape[r];
  size_t e = 1;
  for (int r = 0; r < L.rank; ++r) e *= (size_t)L.shape[r];
  *off = (size_t)L.goff[0] * row;
  *n = e;
}

// the pipelined mdh_execute_host (HostPipe); returns UNSUPPORTED (nothing enqueued) when a
// chunk pointer would be misaligned, so the caller takes the one-shot path
static mdh_status execute_host_pipe(mdh_plan_s* h, const void* const* host_in, void* const* host_out, char* base,
                                    cudaStream_t st) {
  const mdh::Plan& p = h->p;
  HostPipe& P = h->pipe;
  const int C = P.C;
  std::vector<char*> din(p.n_in), dout(p.n_out);
  size_t off = 0;
  for (int b = 0; b < p.n_in; ++b) { din[b] = base + off; off += (host_bytes(p.in[b]) + 255) / 256 * 256; }
  for (int b = 0; b < p.n_out; ++b) { dout[b] = base + off; off += (host_bytes(p.out[b]) + 255) / 256 * 256; }
  char* ws = base + off;
  // chunk slices (element offset, count) and the alignment the kernels need
  std::vector<size_t> io(C * p.n_in), in_n(C * p.n_in), oo(C * p.n_out), on(C * p.n_out);
  std::vector<bool> shared(p.n_in, true);
  for (int c = 0; c < C; ++c) {
    const mdh::Plan& q = P.sub[c]->p;
    for (int b = 0; b < p.n_in; ++b) {
      slice_of(q.in[b], p.in[b], &io[c * p.n_in + b], &in_n[c * p.n_in + b]);
      if (in_n[c * p.n_in + b] != (size_t)p.in[b].elems) shared[b] = false;
      if ((io[c * p.n_in + b] * mdh::dtype_size(p.in[b].dtype)) % 16) return MDH_ERR_UNSUPPORTED;
    }
    for (int b = 0; b < p.n_out; ++b) {
      slice_of(q.out[b], p.out[b], &oo[c * p.n_out + b], &on[c * p.n_out + b]);
      if ((oo[c * p.n_out + b] * mdh::dtype_size(p.out[b].dtype)) % 16) return MDH_ERR_UNSUPPORTED;
    }
  }
  MDH_CUDA(cudaEventRecord(P.ev[0], st));
  MDH_CUDA(cudaStreamWaitEvent(P.s_in, P.ev[0], 0));
  MDH_CUDA(cudaStreamWaitEvent(P.s_out, P.ev[0], 0));
  for (int b = 0; b < p.n_in; ++b)                    // inputs every chunk reads whole: once
    if (shared[b]) MDH_CUDA(cudaMemcpyAsync(din[b], host_in[b], host_bytes(p.in[b]), cudaMemcpyHostToDevice, P.s_in));
  for (int c = 0; c < C; ++c) {
    for (int b = 0; b < p.n_in; ++b) {
      if (shared[b]) continue;
      const size_t es = mdh::dtype_size(p.in[b].dtype), o = io[c * p.n_in + b] * es;
      MDH_CUDA(cudaMemcpyAsync(din[b] + o, (const char*)host_in[b] + o, in_n[c * p.n_in + b] * es,
                               cudaMemcpyHostToDevice, P.s_in));
    }
    MDH_CUDA(cudaEventRecord(P.ev[1 + c], P.s_in));
  }
  if (P.ws_max) MDH_CUDA(cudaMemsetAsync(ws, 0, P.ws_max, st));   // workspace contract
  int launched = 0;
  for (int c = 0; c < C; ++c) {
    MDH_CUDA(cudaStreamWaitEvent(st, P.ev[1 + c], 0));
    const void* ci[MDH_MAX_BUFS];
    void* co[MDH_MAX_BUFS];
    for (int b = 0; b < p.n_in; ++b) ci[b] = din[b] + io[c * p.n_in + b] * mdh::dtype_size(p.in[b].dtype);
    for (int b = 0; b < p.n_out; ++b) co[b] = dout[b] + oo[c * p.n_out + b] * mdh::dtype_size(p.out[b].dtype);
    MDH_TRY(mdh_execute(P.sub[c], ci, co, ws, P.ws_max, st));
    launched += mdh::launch_count();
    MDH_CUDA(cudaEventRecord(P.ev[1 + C + c], st));
  }
  for (int c = 0; c < C; ++c) {
    MDH_CUDA(cudaStreamWaitEvent(P.s_out, P.ev[1 + C + c], 0));
    for (int b = 0; b < p.n_out; ++b) {
      const size_t es = mdh::dtype_size(p.out[b].dtype), o = oo[c * p.n_out + b] * es;
      MDH_CUDA(cudaMemcpyAsync((char*)host_out[b] + o, dout[b] + o, on[c * p.n_out + b] * es, cudaMemcpyDeviceToHost,
                               P.s_out));
    }
  }
  MDH_CUDA(cudaEventRecord(P.ev[2 * C + 1], P.s_out));
  MDH_CUDA(cudaStreamWaitEvent(st, P.ev[2 * C + 1], 0));
  mdh::reset_launch_count();
  mdh::count_launch(launched);
  return MDH_OK;
}

using mdh::set_error;

extern "C" {

mdh_status mdh_plan(const mdh_spec* spec, const mdh_plan_opts* opts, mdh_plan_t* plan_out) {
  if (!plan_out) { set_error("plan_out is NULL"); return MDH_ERR_INVALID_ARG; }
  *plan_out = nullptr;
  mdh_plan_s* h = new (std::nothrow) mdh_plan_s();
  if (!h) { set_error("out of host memory"); return MDH_ERR_OUT_OF_MEMORY; }
  mdh_status s;
  try {
    s = mdh::build_plan(spec, opts, &h->p);
  } catch (...) {
    set_error("internal exception in mdh_plan");
    s = MDH_ERR_INTERNAL;
  }
  if (s != MDH_OK) {
    mdh_destroy(h);
    return s;
  }
  if (spec && (!opts || opts->world_size <= 1) && !h->p.sharded) {
    h->sin.assign(spec->in, spec->in + spec->n_in);
    h->sout.assign(spec->out, spec->out + spec->n_out);
    if (spec->fparams && spec->n_fparams > 0) h->fpar.assign(spec->fparams, spec->fparams + spec->n_fparams);
    h->spec = *spec;
    h->spec.in = h->sin.data();
    h->spec.out = h->sout.data();
    h->spec.fparams = h->fpar.empty() ? nullptr : h->fpar.data();
    if (opts) h->opts = *opts;
    else h->opts.world_size = 1, h->opts.shard_dim = -1;
    if (h->opts.tile_table) h->tile_table = h->opts.tile_table;
    if (h->opts.force_tile) h->force_tile = h->opts.force_tile;
    h->opts.tile_table = h->tile_table.empty() ? nullptr : h->tile_table.c_str();
    h->opts.force_tile = h->force_tile.empty() ? nullptr : h->force_tile.c_str();
    h->have_spec = true;
  }
  *plan_out = h;
  return MDH_OK;
}

mdh_status mdh_plan_workspace_size(mdh_plan_t plan, size_t* bytes) {
  if (!plan || !bytes) { set_error("NULL argument"); return MDH_ERR_INVALID_ARG; }
  *bytes = plan->p.ws_total;
  return MDH_OK;
}

mdh_status mdh_plan_local_shape(mdh_plan_t plan, int32_t is_output, int32_t buf, int64_t* shape,
                                int64_t* global_offset, int32_t* dtype, int32_t* rank) {
  if (!plan) { set_error("NULL plan"); return MDH_ERR_INVALID_ARG; }
  const mdh::Plan& p = plan->p;
  int n = is_output ? p.n_out : p.n_in;
  if (buf < 0 || buf >= n) { set_error("buffer index %d out of range", buf); return MDH_ERR_INVALID_ARG; }
  const mdh::Buf& B = is_output ? p.out[buf] : p.in[buf];
  for (int r = 0; r < MDH_MAX_RANK; ++r) {
    if (shape) shape[r] = r < B.rank ? B.shape[r] : 0;
    if (global_offset) global_offset[r] = r < B.rank ? B.goff[r] : 0;
  }
  if (dtype) *dtype = (int32_t)B.dtype;
  if (rank) *rank = B.rank;
  return MDH_OK;
}

mdh_status mdh_plan_describe(mdh_plan_t plan, char* json, size_t cap, size_t* needed) {
  if (!plan) { set_error("NULL plan"); return MDH_ERR_INVALID_ARG; }
  std::string s = mdh::describe_plan(plan->p);
  if (plan->pipe.ok && !s.empty() && s.back() == '}') {    // the mdh_execute_host pipeline, once built
    s.pop_back();
    s += ", \"host_pipe\": {\"dim\": " + std::to_string(plan->pipe.dim) + ", \"chunks\": " +
         std::to_string(plan->pipe.C) + "}}";
  }
  if (needed) *needed = s.size() + 1;
  if (json && cap > 0) {
    size_t n = std::min(cap - 1, s.size());
    std::memcpy(json, s.data(), n);
    json[n] = 0;
  }
  return MDH_OK;
}

mdh_status mdh_execute(mdh_plan_t plan, const void* const* in, void* const* out, void* workspace,
                       size_t workspace_bytes, void* cuda_stream) {
  mdh::reset_launch_count();
  if (!plan) { set_error("NULL plan"); return MDH_ERR_INVALID_ARG; }
  const mdh::Plan& p = plan->p;
  MDH_TRY(mdh::check_ptrs(p, in, out));
  if (workspace_bytes < p.ws_total || (p.ws_total > 0 && !workspace)) {
    set_error("workspace of %zu bytes is smaller than the %zu the plan needs", workspace_bytes, p.ws_total);
    return MDH_ERR_INVALID_ARG;
  }
  if (workspace && reinterpret_cast<uintptr_t>(workspace) % 256) {
    set_error("workspace must be 256-byte aligned");
    return MDH_ERR_INVALID_ARG;
  }
  cudaStream_t st = (cudaStream_t)cuda_stream;
  try {
    if (p.sharded && p.shard_is_red && p.comm && !(p.flags & MDH_PLAN_NO_COLLECTIVE))
      return mdh::execute_sharded(p, in, out, (char*)workspace, st);
    return mdh::run_template(p, in, out, workspace, st);
  } catch (...) {
    set_error("internal exception in mdh_execute");
    return MDH_ERR_INTERNAL;
  }
}

mdh_status mdh_plan_host_scratch_size(mdh_plan_t plan, size_t* bytes) {
  if (!plan || !bytes) { set_error("NULL argument"); return MDH_ERR_INVALID_ARG; }
  const mdh::Plan& p = plan->p;
  size_t s = 0;
  for (int b = 0; b < p.n_in; ++b) s += ((size_t)p.in[b].elems * mdh::dtype_size(p.in[b].dtype) + 255) / 256 * 256;
  for (int b = 0; b < p.n_out; ++b) s += ((size_t)p.out[b].elems * mdh::dtype_size(p.out[b].dtype) + 255) / 256 * 256;
  ensure_pipe(plan);
  *bytes = s + std::max(p.ws_total, plan->pipe.ok ? plan->pipe.ws_max : (size_t)0) + 256;
  return MDH_OK;
}

mdh_status mdh_execute_host(mdh_plan_t plan, const void* const* host_in, void* const* host_out,
                            void* device_scratch, size_t scratch_bytes, void* cuda_stream) {
  if (!plan || !host_in || !host_out || !device_scratch) { set_error("NULL argument"); return MDH_ERR_INVALID_ARG; }
  const mdh::Plan& p = plan->p;
  size_t need;
  MDH_TRY(mdh_plan_host_scratch_size(plan, &need));
  if (scratch_bytes < need) { set_error("device scratch of %zu bytes < %zu needed", scratch_bytes, need); return MDH_ERR_INVALID_ARG; }
  cudaStream_t st = (cudaStream_t)cuda_stream;
  char* base = (char*)(((uintptr_t)device_scratch + 255) / 256 * 256);
  if (plan->pipe.ok) {                       // chunked: copies in both directions overlap the kernels
    std::lock_guard<std::mutex> g(plan->mu);  // (the plan's copy streams and events)
    const mdh_status ps = execute_host_pipe(plan, host_in, host_out, base, st);
    if (ps != MDH_ERR_UNSUPPORTED) return ps;
  }
  const void* din[MDH_MAX_BUFS];
  void* dout[MDH_MAX_BUFS];
  size_t off = 0;
  int copies = 0;
  for (int b = 0; b < p.n_in; ++b) {
    size_t n = (size_t)p.in[b].elems * mdh::dtype_size(p.in[b].dtype);
    MDH_CUDA(cudaMemcpyAsync(base + off, host_in[b], n, cudaMemcpyHostToDevice, st));
    din[b] = base + off;
    off += (n + 255) / 256 * 256;
    ++copies;
  }
  for (int b = 0; b < p.n_out; ++b) {
    size_t n = (size_t)p.out[b].elems * mdh::dtype_size(p.out[b].dtype);
    dout[b] = base + off;
    off += (n + 255) / 256 * 256;
  }
  void* ws = base + off;
  if (p.ws_total) MDH_CUDA(cudaMemsetAsync(ws, 0, p.ws_total, st));   // workspace contract
  mdh_status s = mdh_execute(plan, din, dout, ws, p.ws_total, cuda_stream);
  if (s != MDH_OK) return s;
  int launched = mdh::launch_count();
  for (int b = 0; b < p.n_out; ++b) {
    size_t n = (size_t)p.out[b].elems * mdh::dtype_size(p.out[b].dtype);
    MDH_CUDA(cudaMemcpyAsync(host_out[b], dout[b], n, cudaMemcpyDeviceToHost, st));
    ++copies;
  }
  mdh::reset_launch_count();
  mdh::count_launch(launched);
  (void)copies;
  return MDH_OK;
}

mdh_status mdh_combine_partials(mdh_plan_t plan, const void* const* partial_outs, int32_t S,
                                void* const* out, void* cuda_stream) {
  mdh::reset_launch_count();
  if (!plan || !partial_outs || !out || S < 1) { set_error("bad arguments"); return MDH_ERR_INVALID_ARG; }
  const mdh::Plan& p = plan->p;
  if (p.nred == 0) { set_error("plan has no pw dimension: partials are concatenated, not combined"); return MDH_ERR_INVALID_ARG; }
  return mdh::launch_combine(p, partial_outs, S, out, (cudaStream_t)cuda_stream);
}

mdh_status mdh_stencil_sweeps(mdh_plan_t plan, void* u, void* v, int32_t sweeps, const mdh_halo* halo,
                              void* workspace, size_t workspace_bytes, void* cuda_stream, int32_t* result_in_v) {
  mdh::reset_launch_count();
  if (!plan || !u || !v || sweeps < 0) { set_error("bad arguments (plan, u, v, sweeps >= 0)"); return MDH_ERR_INVALID_ARG; }
  const mdh::Plan& p = plan->p;
  if (p.n_in != 1 || p.n_out != 1 || p.nred != 0 || p.nps != 0) {
    set_error("stencil sweeps need an all-cc plan with one input and one output buffer");
    return MDH_ERR_INVALID_ARG;
  }
  const mdh::Buf& I = p.in[0];
  const mdh::Buf& O = p.out[0];
  bool same = I.dtype == O.dtype && I.rank == O.rank && I.elems == O.elems;
  for (int r = 0; same && r < I.rank; ++r) same = I.shape[r] == O.shape[r];
  if (!same || I.rank < 2) {
    set_error("stencil sweeps: input and output buffers must have the same dtype and shape (rank >= 2)");
    return MDH_ERR_INVALID_ARG;
  }
  {  // alignment and aliasing of u / v (reading C-27), as mdh_execute checks them
    const void* ins[1] = {u};
    void* outs[1] = {v};
    MDH_TRY(mdh::check_ptrs(p, ins, outs));
  }
  const int64_t nz = I.shape[0];
  const size_t plane = (size_t)(I.elems / nz) * mdh::dtype_size(I.dtype);
  const int world = halo ? halo->world : 1, rank = halo ? halo->rank : 0;
  if (world < 1 || rank < 0 || rank >= world) { set_error("bad halo rank/world"); return MDH_ERR_INVALID_ARG; }
  const bool nccl = world > 1 && halo->nccl_comm;
  if (world > 1 && nz < 3) { set_error("a slab needs >= 3 planes (halo, owned, halo)"); return MDH_ERR_INVALID_ARG; }
  if (world > 1 && !nccl) {
    if ((rank > 0 && (!halo->peer_lo[0] || !halo->peer_lo[1])) ||
        (rank < world - 1 && (!halo->peer_hi[0] || !halo->peer_hi[1]))) {
      set_error("stencil sweeps: world > 1 needs nccl_comm or the neighbours' halo-plane addresses");
      return MDH_ERR_INVALID_ARG;
    }
    // the peer transport has no cross-rank wait: sweep t+1 would read halo planes the
    // neighbours' sweep t has not written yet, so the caller steps the ranks one sweep
    // per call in lock-step
    if (sweeps > 1) {
      set_error("stencil sweeps: the peer transport runs one sweep per call (lock-step); use nccl_comm for more");
      return MDH_ERR_INVALID_ARG;
    }
    const size_t esz = mdh::dtype_size(I.dtype);
    for (int k = 0; k < 2; ++k) {
      const void* q[2] = {halo->peer_lo[k], halo->peer_hi[k]};
      for (const void* a : q)
        if (a && reinterpret_cast<uintptr_t>(a) % esz) {
          set_error("stencil sweeps: a peer halo-plane address is not %zu-byte aligned", esz);
          return MDH_ERR_INVALID_ARG;
        }
      // a neighbour's halo plane must not lie inside this rank's own u / v
      for (const void* a : q) {
        if (!a) continue;
        const uintptr_t h0 = (uintptr_t)a, h1 = h0 + plane;
        for (const void* b : {(const void*)u, (const void*)v}) {
          const uintptr_t b0 = (uintptr_t)b, b1 = b0 + (uintptr_t)I.elems * esz;
          if (h0 < b1 && b0 < h1) {
            set_error("stencil sweeps: a peer halo plane overlaps this rank's u or v");
            return MDH_ERR_INVALID_ARG;
          }
        }
      }
    }
  }
  cudaStream_t st = (cudaStream_t)cuda_stream;
  char* buf[2] = {(char*)u, (char*)v};
  int launches = 0;
  for (int t = 0; t < sweeps; ++t) {
    const int s = t & 1, d = s ^ 1;
    const void* in[1] = {buf[s]};
    void* out[1] = {buf[d]};
    if (world == 1 || !nccl) {
      // one 7-point kernel per sweep, sweep t > 0 launched as a programmatic dependent of
      // sweep t-1; peer transport: the kernel also stores its first / last plane straight
      // into the neighbours' halo planes (no copies)
      mdh::reset_launch_count();
      mdh_status e = mdh::launch_t1_halo(p, buf[s], buf[d], world > 1 && rank > 0 ? halo->peer_lo[d] : nullptr,
                                         world > 1 && rank < world - 1 ? halo->peer_hi[d] : nullptr, st, t > 0);
      if (e == MDH_OK) {
        launches += mdh::launch_count();
        continue;
      }
      if (e != MDH_ERR_UNSUPPORTED) return e;
    }
    mdh_status e = mdh_execute(plan, in, out, workspace, workspace_bytes, cuda_stream);
    if (e != MDH_OK) return e;
    launches += mdh::launch_count();
    if (world > 1) {
      if (nccl) {
        MDH_TRY(mdh::comm_halo_exchange(halo->nccl_comm, rank, world, buf[d], plane, nz, st));
      } else {
        if (rank > 0) MDH_CUDA(cudaMemcpyAsync(halo->peer_lo[d], buf[d] + plane, plane, cudaMemcpyDeviceToDevice, st));
        if (rank < world - 1)
          MDH_CUDA(cudaMemcpyAsync(halo->peer_hi[d], buf[d] + (nz - 2) * plane, plane, cudaMemcpyDeviceToDevice, st));
      }
    }
  }
  mdh::reset_launch_count();
  mdh::count_launch(launches);
  if (result_in_v) *result_in_v = sweeps & 1;
  return MDH_OK;
}

mdh_status mdh_destroy(mdh_plan_t plan) {
  if (!plan) return MDH_OK;
  if (plan->p.dconst) {
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(plan->p.device);
    cudaFree(plan->p.dconst);
    cudaSetDevice(cur);
  }
  mdh::release_t4(&plan->p);
  for (auto q : plan->pipe.sub) mdh_destroy(q);
  for (auto e : plan->pipe.ev)
    if (e) cudaEventDestroy(e);
  if (plan->pipe.s_in) cudaStreamDestroy(plan->pipe.s_in);
  if (plan->pipe.s_out) cudaStreamDestroy(plan->pipe.s_out);
  delete plan;
  return MDH_OK;
}

mdh_status mdh_comm_unique_id(void* id128) { return mdh::comm_unique_id(id128); }
mdh_status mdh_comm_init(const void* id128, int32_t world, int32_t rank, int32_t device, void** comm_out) {
  return mdh::comm_init(id128, world, rank, device, comm_out);
}
mdh_status mdh_comm_destroy(void* comm) { return mdh::comm_destroy(comm); }

mdh_status mdh_measure_peaks(int32_t device, double* ffma_tflops, double* alu_tops, double* issue_tops) {
  return mdh::measure_peaks(device, ffma_tflops, alu_tops, issue_tops);
}

const char* mdh_last_error(void) { return mdh::g_err.c_str(); }
int32_t mdh_abi_version(void) { return MDH_ABI_VERSION; }
int32_t mdh_last_launch_count(void) { return mdh::launch_count(); }

}  // extern "C"
