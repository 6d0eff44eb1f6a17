// planner.cpp — mdh_plan: validation, dimension classification, template choice,
// multi-GPU sub-domain rewrite.
//
// Validation follows the readings of DESIGN.md §3: sizes >= 1 (C-10), affine index
// functions with non-negative coordinates (C-8), declared shapes containing every
// access or inferred as max+1 (fn.7 P:316, C-9), injective outputs (C-5), one common
// pw operator (C-3), f arity per the catalog.
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <numeric>
#include <string>
#include <vector>

#include "internal.h"

namespace mdh {

const char* template_name(int t) {
  switch (t) {
    case T0_GENERIC: return "T0_generic";
    case T1_STENCIL: return "T1_stencil";
    case T2_REDUCE: return "T2_reduce";
    case T3_SIMT: return "T3_simt_contraction";
    case T4_TC: return "T4_tcgen05_contraction";
    case T5_PRL: return "T5_prl_pairwise";
    case T6_SCAN: return "T6_prefix_scan";
  }
  return "?";
}

static bool valid_dtype(int t) { return t >= MDH_BF16 && t <= MDH_I64; }

// range of coordinate r of index fn `fn` over the box `size`; pw dims fixed to 0 when
// `collapse_red` (output index functions, reading C-4).
static void coord_range(const Plan& p, const mdh_index_fn& fn, int r, bool collapse_red,
                        int64_t* lo, int64_t* hi) {
  int64_t l = fn.offset[r], h = fn.offset[r];
  for (int d = 0; d < p.D; ++d) {
    // output index functions see pw indices = 0 (C-4); cc and ps indices are kept
    int64_t ext = (collapse_red && p.op[d] != MDH_CC && p.op[d] != MDH_PS_ADD) ? 0 : p.size[d] - 1;
    int64_t c = fn.coeff[r][d];
    if (c > 0) h += c * ext; else l += c * ext;
  }
  *lo = l;
  *hi = h;
}

static void linearise(const Plan& p, Buf* B) {
  int64_t stride[MDH_MAX_RANK];
  int64_t s = 1;
  for (int r = B->rank - 1; r >= 0; --r) {
    stride[r] = s;
    s *= B->shape[r];
  }
  B->elems = s;
  for (int a = 0; a < B->nacc; ++a) {
    Access& A = B->acc[a];
    A.base = 0;
    for (int d = 0; d < MDH_MAX_D; ++d) A.L[d] = 0;
    for (int r = 0; r < B->rank; ++r) {
      A.base += B->fn[a].offset[r] * stride[r];
      for (int d = 0; d < p.D; ++d) A.L[d] += B->fn[a].coeff[r][d] * stride[r];
    }
  }
}

// Injectivity of the output map over the cc sub-box (reading C-5).  A mixed-radix
// argument proves it for one access; otherwise a bitmap check for small outputs.
static mdh_status check_injective(const Plan& p, const Buf& B, int b) {
  if (B.nacc == 1) {
    std::vector<std::pair<int64_t, int64_t>> v;
    for (int t = 0; t < p.ncc; ++t) {
      int d = p.cc[t];
      if (p.size[d] <= 1) continue;
      int64_t L = B.acc[0].L[d] < 0 ? -B.acc[0].L[d] : B.acc[0].L[d];
      if (L == 0) {
        set_error("output %d: index function ignores cc dim %d, so cc points collide "
                  "(not injective, reading C-5)", b, d);
        return MDH_ERR_INVALID_SPEC;
      }
      v.push_back({L, p.size[d]});
    }
    std::sort(v.begin(), v.end());
    int64_t reach = 0;
    bool ok = true;
    for (auto& e : v) {
      if (e.first <= reach) { ok = false; break; }
      reach += e.first * (e.second - 1);
    }
    if (ok) return MDH_OK;
  }
  // bitmap fallback (host, plan time)
  int64_t npts = 1;
  for (int t = 0; t < p.ncc; ++t) npts *= p.size[p.cc[t]];
  if (npts * B.nacc > (int64_t(1) << 26) || B.elems > (int64_t(1) << 30)) {
    set_error("output %d: cannot prove the output index functions injective", b);
    return MDH_ERR_UNSUPPORTED;
  }
  std::vector<uint8_t> mark((size_t)B.elems, 0);
  int64_t idx[MDH_MAX_D] = {0};
  for (int64_t q = 0; q < npts; ++q) {
    int64_t rem = q;
    for (int t = p.ncc - 1; t >= 0; --t) {
      idx[p.cc[t]] = rem % p.size[p.cc[t]];
      rem /= p.size[p.cc[t]];
    }
    for (int a = 0; a < B.nacc; ++a) {
      int64_t k = B.acc[a].base;
      for (int t = 0; t < p.ncc; ++t) k += B.acc[a].L[p.cc[t]] * idx[p.cc[t]];
      if (mark[(size_t)k]) {
        set_error("output %d: two cc points write the same element (not injective, C-5)", b);
        return MDH_ERR_INVALID_SPEC;
      }
      mark[(size_t)k] = 1;
    }
  }
  return MDH_OK;
}

static mdh_status copy_buffer(const Plan& p, const mdh_buffer& src, Buf* B, bool is_out, int b) {
  if (!valid_dtype(src.dtype)) { set_error("buffer %d: bad dtype", b); return MDH_ERR_INVALID_SPEC; }
  if (src.rank < 1 || src.rank > MDH_MAX_RANK) { set_error("buffer %d: rank %d out of [1,%d]", b, src.rank, MDH_MAX_RANK); return MDH_ERR_INVALID_SPEC; }
  if (src.n_acc < 1 || src.n_acc > MDH_MAX_ACC) { set_error("buffer %d: %d accesses", b, src.n_acc); return MDH_ERR_INVALID_SPEC; }
  B->dtype = src.dtype;
  B->rank = src.rank;
  B->nacc = src.n_acc;
  for (int a = 0; a < src.n_acc; ++a) {
    B->fn[a] = src.acc[a];
    for (int r = src.rank; r < MDH_MAX_RANK; ++r) {
      B->fn[a].offset[r] = 0;
      for (int d = 0; d < MDH_MAX_D; ++d) B->fn[a].coeff[r][d] = 0;
    }
    for (int r = 0; r < src.rank; ++r)
      for (int d = p.D; d < MDH_MAX_D; ++d) B->fn[a].coeff[r][d] = 0;
  }
  bool declared = false;
  for (int r = 0; r < src.rank; ++r) declared |= src.shape[r] != 0;
  for (int r = 0; r < MDH_MAX_RANK; ++r) { B->shape[r] = 0; B->goff[r] = 0; }
  for (int r = 0; r < src.rank; ++r) {
    int64_t mx = -1;
    for (int a = 0; a < src.n_acc; ++a) {
      int64_t lo, hi;
      coord_range(p, B->fn[a], r, is_out, &lo, &hi);
      if (lo < 0) {
        set_error("%s buffer %d access %d: coordinate %d can be negative (%lld)",
                  is_out ? "output" : "input", b, a, r, (long long)lo);
        return MDH_ERR_INVALID_SPEC;
      }
      mx = std::max(mx, hi);
    }
    if (declared) {
      if (src.shape[r] <= mx) {
        set_error("%s buffer %d: declared shape[%d]=%lld does not contain accessed index %lld "
                  "(fn.7 P:316)", is_out ? "output" : "input", b, r, (long long)src.shape[r], (long long)mx);
        return MDH_ERR_INVALID_SPEC;
      }
      B->shape[r] = src.shape[r];
    } else {
      B->shape[r] = mx + 1;
    }
  }
  for (int r = 0; r < MDH_MAX_RANK; ++r) B->gshape[r] = B->shape[r];
  return MDH_OK;
}

// ---- multi-GPU sub-domain rewrite ------------------------------
static void partition(int64_t n, int world, int rank, int64_t* start, int64_t* len) {
  int64_t base = n / world, rem = n % world;
  *len = base + (rank < rem ? 1 : 0);
  *start = rank * base + std::min<int64_t>(rank, rem);
}

static mdh_status shard_rewrite(Plan* p) {
  int d = p->shard_dim;
  p->global_size = p->size[d];
  partition(p->size[d], p->world, p->rank, &p->shard_start, &p->shard_len);
  if (p->shard_len < 1) {
    set_error("shard dim %d of size %lld cannot be split over %d ranks (reading C-10)", d,
              (long long)p->size[d], p->world);
    return MDH_ERR_INVALID_ARG;
  }
  p->size[d] = p->shard_len;
  p->shard_is_red = p->op[d] != MDH_CC;
  auto rewrite = [&](Buf* B, bool is_out) {
    if (is_out && p->shard_is_red) return;        // collapsed index stays 0 (C-4)
    for (int a = 0; a < B->nacc; ++a)
      for (int r = 0; r < B->rank; ++r) B->fn[a].offset[r] += B->fn[a].coeff[r][d] * p->shard_start;
    // local origin: coordinates that depend on the shard dim are cut to the accessed range
    for (int r = 0; r < B->rank; ++r) {
      bool dep = false;
      for (int a = 0; a < B->nacc; ++a) dep |= B->fn[a].coeff[r][d] != 0;
      if (!dep) continue;
      int64_t lo = INT64_MAX, hi = -1;
      for (int a = 0; a < B->nacc; ++a) {
        int64_t l, h;
        coord_range(*p, B->fn[a], r, is_out, &l, &h);
        lo = std::min(lo, l);
        hi = std::max(hi, h);
      }
      B->goff[r] = lo;
      B->shape[r] = hi - lo + 1;
      for (int a = 0; a < B->nacc; ++a) B->fn[a].offset[r] -= lo;
    }
  };
  for (int b = 0; b < p->n_in; ++b) rewrite(&p->in[b], false);
  for (int b = 0; b < p->n_out; ++b) rewrite(&p->out[b], true);
  return MDH_OK;
}

static int choose_shard_dim(const Plan& p) {
  if (p.f == MDH_F_PRL_COMPARE && p.nred > 0) return p.red[0];   // §8(e): PRL shards the DB dim
  for (int t = 0; t < p.ncc; ++t)
    if (p.op[p.cc[t]] == MDH_CC && p.size[p.cc[t]] >= p.world) return p.cc[t];
  for (int t = 0; t < p.nred; ++t)
    if (p.op[p.red[t]] != MDH_PS_ADD && p.size[p.red[t]] >= p.world) return p.red[t];
  return -1;
}

// ---- contraction grouping (A0): M = dims only A uses, N = only B, batch = both -------
static bool group_contraction(Plan* p) {
  if (p->nps > 0 || p->f != MDH_F_MUL || p->n_in != 2 || p->in[0].nacc != 1 || p->in[1].nacc != 1) return false;
  if (p->nred == 0 || p->redop != MDH_PW_ADD) return false;
  Contraction c;
  const Access& A = p->in[0].acc[0];
  const Access& B = p->in[1].acc[0];
  for (int d = 0; d < p->D; ++d) {
    if (p->size[d] == 1) continue;     // degenerate dims carry no work
    bool ua = A.L[d] != 0, ub = B.L[d] != 0;
    if (p->op[d] != MDH_CC) {
      c.kd[c.nk++] = d;
      c.K *= p->size[d];
    } else if (ua && ub) {
      c.zd[c.nz++] = d;
      c.Z *= p->size[d];
    } else if (ua) {
      c.md[c.nm++] = d;
      c.M *= p->size[d];
    } else if (ub) {
      c.nd[c.nn++] = d;
      c.N *= p->size[d];
    } else {
      return false;                    // a cc dim neither operand uses: output broadcast
    }
  }
  if (c.nm == 0 || c.nn == 0 || c.nk == 0) return false;
  // enumerate each group with the output's most contiguous dim fastest, so that
  // consecutive m (n) are as close as possible in the output (coalesced epilogues)
  const Access& Co = p->out[0].acc[0];
  auto by_out_stride = [&](int* dims, int n) {
    std::stable_sort(dims, dims + n, [&](int x, int y) {
      int64_t lx = Co.L[x] < 0 ? -Co.L[x] : Co.L[x], ly = Co.L[y] < 0 ? -Co.L[y] : Co.L[y];
      return lx > ly;
    });
  };
  by_out_stride(c.md, c.nm);
  by_out_stride(c.nd, c.nn);
  by_out_stride(c.zd, c.nz);
  // orientation: the output's most contiguous dim goes to the N group (TMEM columns in T4,
  // the thread-x direction in T3), so a thread's consecutive accumulators are consecutive
  // output elements and the epilogue stores vectors.  f = MUL is commutative (x0·x1 =
  // x1·x0 exactly), so A/B may swap (CCSD(T): t3's unit-stride p4 is a t2 dim)
  auto min_stride = [&](const int* dims, int n) {
    int64_t s = INT64_MAX;
    for (int t = 0; t < n; ++t) s = std::min(s, Co.L[dims[t]] < 0 ? -Co.L[dims[t]] : Co.L[dims[t]]);
    return s;
  };
  if (min_stride(c.md, c.nm) < min_stride(c.nd, c.nn)) {
    int tmp[MDH_MAX_D];
    std::copy(c.md, c.md + c.nm, tmp);
    std::copy(c.nd, c.nd + c.nn, c.md);
    std::copy(tmp, tmp + c.nm, c.nd);
    std::swap(c.nm, c.nn);
    std::swap(c.M, c.N);
    c.a_buf = 1;
    c.b_buf = 0;
  }
  p->con = c;
  return true;
}

static mdh_status select_template(Plan* p) {
  char buf[256];
  // compute type (reading C-13 / C-12)
  bool allf = true, alli = true, any64 = false, anyi64 = false;
  for (int b = 0; b < p->n_in; ++b) {
    if (is_float(p->in[b].dtype)) alli = false; else allf = false;
    any64 |= p->in[b].dtype == MDH_F64;
    anyi64 |= p->in[b].dtype == MDH_I64;
  }
  if (p->f == MDH_F_PRL_COMPARE) {
    p->compute = MDH_F64;
  } else if (allf) {
    p->compute = any64 ? MDH_F64 : MDH_F32;
  } else if (alli) {
    if (anyi64) {
      for (int b = 0; b < p->n_in; ++b)
        if (p->in[b].dtype != MDH_I64) { set_error("mixed int64/int32 inputs"); return MDH_ERR_UNSUPPORTED; }
      p->compute = MDH_I64;
    } else {
      mdh_dtype t0 = p->in[0].dtype;
      for (int b = 0; b < p->n_in; ++b)
        if (p->in[b].dtype != t0) { set_error("mixed int32/uint32 inputs"); return MDH_ERR_UNSUPPORTED; }
      p->compute = t0;
    }
  } else {
    set_error("mixed integer and floating-point inputs are outside the catalog");
    return MDH_ERR_UNSUPPORTED;
  }
  if (p->f != MDH_F_PRL_COMPARE) {
    mdh_dtype ot = p->out[0].dtype;
    if (is_float(p->compute) != is_float(ot)) {
      set_error("output dtype does not match the arithmetic type of f");
      return MDH_ERR_UNSUPPORTED;
    }
    if (p->compute == MDH_F64 && ot != MDH_F64) {
      set_error("f64 inputs need an f64 output");
      return MDH_ERR_UNSUPPORTED;
    }
  }
  if (p->f == MDH_F_STENCIL && !allf) { set_error("STENCIL needs floating-point inputs"); return MDH_ERR_UNSUPPORTED; }

  // template choice (SURVEY §8(a) A0 decision table)
  p->tmpl = T0_GENERIC;
  p->why = "generic fallback";
  if (p->nps > 0) {
    p->tmpl = T6_SCAN;
    p->why = "ps(add) dim: prefix-sum scan";
  } else if (p->f == MDH_F_PRL_COMPARE) {
    p->tmpl = T5_PRL;
    p->why = "f = PRL_COMPARE";
  } else if (p->nred == 0) {
    p->tmpl = T1_STENCIL;
    p->why = "RED = {} (all cc): map/stencil";
  } else if (group_contraction(p)) {
    std::string w;
    bool bf = p->in[0].dtype == MDH_BF16 && p->in[1].dtype == MDH_BF16;
    if (bf && t4_supported(*p, &w)) {
      p->tmpl = T4_TC;
      p->why = "f=MUL, ⊗=pw(add), M and N non-empty, bf16: tcgen05 (" + w + ")";
    } else if (p->compute == MDH_F32 || p->compute == MDH_I32 || p->compute == MDH_U32) {
      p->tmpl = T3_SIMT;
      std::snprintf(buf, sizeof(buf), "f=MUL, ⊗=pw(add), M=%lld N=%lld K=%lld Z=%lld: SIMT contraction%s%s",
                    (long long)p->con.M, (long long)p->con.N, (long long)p->con.K, (long long)p->con.Z,
                    bf ? "; tcgen05 rejected: " : "", bf ? w.c_str() : "");
      p->why = buf;
    }
  }
  if (p->tmpl == T0_GENERIC && p->nred > 0 && (p->f == MDH_F_MUL || p->f == MDH_F_IDENTITY) &&
      (p->redop == MDH_PW_ADD || p->redop == MDH_PW_MAX || p->redop == MDH_PW_MIN)) {
    p->tmpl = T2_REDUCE;
    p->why = "pw reduction with little reuse: streaming reduction";
  }
  return MDH_OK;
}

mdh_status build_plan(const mdh_spec* spec, const mdh_plan_opts* opts, Plan* p) {
  if (!spec) { set_error("spec is NULL"); return MDH_ERR_INVALID_ARG; }
  if (spec->D < 1 || spec->D > MDH_MAX_D) { set_error("D=%d out of [1,%d]", spec->D, MDH_MAX_D); return MDH_ERR_INVALID_SPEC; }
  p->D = spec->D;
  for (int d = 0; d < p->D; ++d) {
    if (spec->size[d] < 1) {
      set_error("size of dim %d is %lld; sizes must be >= 1 (reading C-10)", d, (long long)spec->size[d]);
      return MDH_ERR_INVALID_SPEC;
    }
    if ((int)spec->op[d] < MDH_CC || (int)spec->op[d] > MDH_PS_ADD) {
      set_error("dim %d: unknown combine operator %d", d, (int)spec->op[d]);
      return MDH_ERR_UNSUPPORTED;
    }
    p->size[d] = spec->size[d];
    p->op[d] = spec->op[d];
  }
  for (int d = p->D; d < MDH_MAX_D; ++d) { p->size[d] = 1; p->op[d] = MDH_CC; }
  if ((int)spec->f < MDH_F_MUL || (int)spec->f > MDH_F_IDENTITY) { set_error("unknown f"); return MDH_ERR_UNSUPPORTED; }
  p->f = spec->f;
  if (spec->n_fparams < 0 || (spec->n_fparams > 0 && !spec->fparams)) { set_error("bad fparams"); return MDH_ERR_INVALID_ARG; }
  p->fparams.assign(spec->fparams, spec->fparams + spec->n_fparams);
  if (spec->n_in < 1 || spec->n_out < 1 || spec->n_in + spec->n_out > MDH_MAX_BUFS || !spec->in || !spec->out) {
    set_error("need >=1 input and >=1 output buffer, at most %d in total", MDH_MAX_BUFS);
    return MDH_ERR_INVALID_SPEC;
  }
  p->n_in = spec->n_in;
  p->n_out = spec->n_out;
  // classification
  p->ncc = p->nred = 0;
  p->redop = MDH_CC;
  p->nps = 0;
  for (int d = 0; d < p->D; ++d) {
    if (p->op[d] == MDH_CC) p->cc[p->ncc++] = d;
    else if (p->op[d] == MDH_PS_ADD) {
      // a ps dim is kept in the result (enumerated like cc) and folded over [0, k]
      p->cc[p->ncc++] = d;
      p->red[p->nred++] = d;
      p->ps[p->nps++] = d;
    } else {
      if (p->redop != MDH_CC && p->op[d] != p->redop) {
        set_error("dims use different pw operators; the result would depend on the split "
                  "(interchange law fails, reading C-3)");
        return MDH_ERR_UNSUPPORTED;
      }
      p->redop = p->op[d];
      p->red[p->nred++] = d;
    }
  }
  if (p->nps > 0) {
    if (p->redop != MDH_CC && p->redop != MDH_PW_ADD) {
      set_error("ps(add) combines only with pw(add) dims (interchange law, reading C-3)");
      return MDH_ERR_UNSUPPORTED;
    }
    if (spec->f == MDH_F_PRL_COMPARE) { set_error("ps with PRL_COMPARE is outside the catalog"); return MDH_ERR_UNSUPPORTED; }
    p->redop = MDH_PW_ADD;
  }
  bool prl_op = p->redop == MDH_PW_PRL_ARGMAX || p->redop == MDH_PW_PRL_PAPER;
  if (prl_op != (p->f == MDH_F_PRL_COMPARE) && !(p->f == MDH_F_PRL_COMPARE && p->nred == 0)) {
    set_error("the PRL combine operators go with f = PRL_COMPARE only");
    return MDH_ERR_UNSUPPORTED;
  }
  for (int b = 0; b < p->n_in; ++b) MDH_TRY(copy_buffer(*p, spec->in[b], &p->in[b], false, b));
  for (int b = 0; b < p->n_out; ++b) MDH_TRY(copy_buffer(*p, spec->out[b], &p->out[b], true, b));
  // arity (P:435 SF signature; catalog)
  int nin_acc = 0, nout_acc = 0;
  for (int b = 0; b < p->n_in; ++b) nin_acc += p->in[b].nacc;
  for (int b = 0; b < p->n_out; ++b) nout_acc += p->out[b].nacc;
  p->n_in_acc = nin_acc;
  switch (p->f) {
    case MDH_F_MUL:
      if (nin_acc != 2 || nout_acc != 1) { set_error("MUL takes 2 input accesses and 1 output access"); return MDH_ERR_INVALID_SPEC; }
      break;
    case MDH_F_IDENTITY:
      if (nin_acc != 1 || nout_acc != 1) { set_error("IDENTITY takes 1 input access and 1 output access"); return MDH_ERR_INVALID_SPEC; }
      break;
    case MDH_F_STENCIL:
      if (nout_acc != 1 || nin_acc != (int)p->fparams.size() || nin_acc > 32) {
        set_error("STENCIL takes n<=32 input accesses, n weights (fparams) and 1 output access");
        return MDH_ERR_INVALID_SPEC;
      }
      break;
    case MDH_F_PRL_COMPARE: {
      if (nin_acc != 17 || p->n_in != 17 || p->n_out != 3 || nout_acc != 3 || p->fparams.size() != 16) {
        set_error("PRL_COMPARE takes 8 new-record fields, 8 DB fields, db_id, 16 weights and 3 outputs");
        return MDH_ERR_INVALID_SPEC;
      }
      for (int b = 0; b < 16; ++b)
        if (p->in[b].dtype != MDH_U32) { set_error("PRL fields must be u32 codes (reading C-18)"); return MDH_ERR_UNSUPPORTED; }
      if (p->in[16].dtype != MDH_I64 || p->out[0].dtype != MDH_I64 || p->out[1].dtype != MDH_F64 ||
          p->out[2].dtype != MDH_I32) {
        set_error("PRL types: db_id/match_id int64, match_weight fp64, id_measure int32 (Listing 11)");
        return MDH_ERR_UNSUPPORTED;
      }
      break;
    }
  }
  // multi-GPU
  p->device = opts ? opts->device : 0;
  p->world = opts ? std::max(1, opts->world_size) : 1;
  p->rank = opts ? opts->rank : 0;
  p->flags = opts ? opts->flags : 0;
  p->comm = opts ? opts->nccl_comm : nullptr;
  if (p->world > MDH_MAX_WORLD || p->rank < 0 || p->rank >= p->world) {
    set_error("rank %d / world %d invalid", p->rank, p->world);
    return MDH_ERR_INVALID_ARG;
  }
  // a one-rank plan with a communicator and an explicit shard dim runs the sharded path too
  // (its collective over the one-rank NCCL communicator): the NCCL data plane on one GPU
  if (p->world > 1 || (p->comm && opts->shard_dim >= 0)) {
    p->sharded = true;
    int sd = opts->shard_dim >= 0 ? opts->shard_dim : choose_shard_dim(*p);
    if (sd < 0 || sd >= p->D) { set_error("no dimension can be sharded over %d ranks", p->world); return MDH_ERR_INVALID_ARG; }
    if (p->size[sd] < p->world) { set_error("shard dim %d has %lld < %d points", sd, (long long)p->size[sd], p->world); return MDH_ERR_INVALID_ARG; }
    if (p->op[sd] == MDH_PS_ADD) { set_error("sharding a ps dim is not supported in this build"); return MDH_ERR_UNSUPPORTED; }
    p->shard_dim = sd;
    if (p->op[sd] != MDH_CC && !(p->flags & (MDH_PLAN_VIRTUAL_SHARD | MDH_PLAN_NO_COLLECTIVE)) && !p->comm) {
      set_error("a pw shard needs an NCCL communicator (mdh_comm_init) or MDH_PLAN_VIRTUAL_SHARD");
      return MDH_ERR_INVALID_ARG;
    }
    MDH_TRY(shard_rewrite(p));
  }
  // linearise + per-buffer checks on the local problem
  for (int b = 0; b < p->n_in; ++b) linearise(*p, &p->in[b]);
  for (int b = 0; b < p->n_out; ++b) linearise(*p, &p->out[b]);
  p->Ncc = 1;
  p->Nred = 1;
  for (int t = 0; t < p->ncc; ++t) p->Ncc *= p->size[p->cc[t]];
  for (int t = 0; t < p->nred; ++t) p->Nred *= p->size[p->red[t]];
  for (int b = 0; b < p->n_out; ++b) MDH_TRY(check_injective(*p, p->out[b], b));
  MDH_TRY(select_template(p));
  lookup_tiles(p, opts ? opts->tile_table : nullptr, opts ? opts->force_tile : nullptr);
  switch (p->tmpl) {
    case T0_GENERIC: MDH_TRY(prepare_t0(p)); break;
    case T1_STENCIL: MDH_TRY(prepare_t1(p)); break;
    case T2_REDUCE: MDH_TRY(prepare_t2(p)); break;
    case T3_SIMT: MDH_TRY(prepare_t3(p)); break;
    case T4_TC: MDH_TRY(prepare_t4(p)); break;
    case T5_PRL: MDH_TRY(prepare_t5(p)); break;
    case T6_SCAN: MDH_TRY(prepare_t6(p)); break;
  }
  // pw shard: room for the gathered partials of all ranks
  p->ws_comm = 0;
  if (p->sharded && p->shard_is_red && p->comm && !(p->flags & MDH_PLAN_NO_COLLECTIVE)) {
    size_t per = 0;
    for (int b = 0; b < p->n_out; ++b) per += ((size_t)p->out[b].elems * dtype_size(p->out[b].dtype) + 255) / 256 * 256;
    p->ws_comm = per * (size_t)(p->world + 1);
  }
  p->ws_kernel = (p->ws_kernel + 255) / 256 * 256;
  p->ws_total = p->ws_kernel + p->ws_comm;
  return MDH_OK;
}

std::string describe_plan(const Plan& p) {
  std::string s = "{";
  char b[512];
  auto add = [&](const char* fmt, auto... a) { std::snprintf(b, sizeof(b), fmt, a...); s += b; };
  add("\"template\": \"%s\", \"template_id\": %d, \"why\": \"", template_name(p.tmpl), p.tmpl);
  for (char c : p.why) { if (c == '"') s += '\''; else s += c; }
  s += "\"";
  add(", \"D\": %d, \"Ncc\": %lld, \"Nred\": %lld, \"compute\": %d", p.D, (long long)p.Ncc, (long long)p.Nred, (int)p.compute);
  s += ", \"cc\": [";
  for (int t = 0; t < p.ncc; ++t) add("%s%d", t ? ", " : "", p.cc[t]);
  s += "], \"red\": [";
  for (int t = 0; t < p.nred; ++t) add("%s%d", t ? ", " : "", p.red[t]);
  s += "]";
  if (p.tmpl == T3_SIMT || p.tmpl == T4_TC)
    add(", \"contraction\": {\"Z\": %lld, \"M\": %lld, \"N\": %lld, \"K\": %lld, \"nm\": %d, \"nn\": %d, \"nk\": %d, \"nz\": %d}",
        (long long)p.con.Z, (long long)p.con.M, (long long)p.con.N, (long long)p.con.K, p.con.nm, p.con.nn, p.con.nk, p.con.nz);
  add(", \"tiles\": {\"threads\": %d, \"bm\": %d, \"bn\": %d, \"bk\": %d, \"split\": %d, \"stages\": %d, \"vec\": %d, "
      "\"zchunk\": %d, \"per_thread\": %d, \"cluster\": %d, \"implicit\": %d, \"seg\": %d, \"epi\": %d, \"mode\": %d, "
      "\"source\": \"%s\"}",
      p.tiles.threads, p.tiles.bm, p.tiles.bn, p.tiles.bk, p.tiles.split, p.tiles.stages, p.tiles.vec,
      p.tiles.zchunk, p.tiles.per_thread, p.tiles.cluster, p.tiles.implicit, p.tiles.seg, p.tiles.epi, p.tiles.mode,
      p.tiles.source.c_str());
  add(", \"t4_variant\": %d", p.t4_variant);
  add(", \"workspace\": %zu, \"world\": %d, \"rank\": %d, \"shard_dim\": %d, \"shard_is_red\": %s, "
      "\"shard_start\": %lld, \"shard_len\": %lld}",
      p.ws_total, p.world, p.rank, p.shard_dim, p.shard_is_red ? "true" : "false",
      (long long)p.shard_start, (long long)p.shard_len);
  return s;
}

}  // namespace mdh
