/*
 * mdh_oracle.c — CPU ORACLE for the MDH hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  It shares no code, header, table or constant with the
 * CUDA path (paper_conf_sc_schulzegr25_b200/) and includes nothing from it; it has
 * its own spec encoding (written by oracle/oracle.py) and its own catalog functions.
 *
 * What it computes — the plain definition of md_hom, evaluated literally:
 *
 *   fn.2:  ⊗_1 over i_1 … ⊗_D over i_D  f(a[i_1..i_D])
 *   inp_view:  x(i) = ( in_b[ ι_{b,a}(i) ] )  in (buffer, access) order
 *   md_hom    (Listing 7):  y(i) = f(x(i))
 *   cc        (Listing 15):   places each operand at its own index
 *   pw(cf)    (Listing 16):   cf at every point of the other dims, into index 0
 *   out_view:  out_b[ ω_{b,a}(j) ] := R[j], pw indices = 0 (reading C-4)
 *
 * Algorithm: for every cc coordinate j (lexicographic, dimension
 * order), R[j] = FOLD over the pw dims, outermost pw dim first (reading C-1); each
 * pw is a LEFT fold over ascending indices starting from index 0, the lhs always
 * being the lower index range (Listing 16's (lhs, rhs) = (P, Q); reading C-2).
 *
 * Arithmetic (reading C-13, C-12): fp32/bf16 inputs are widened exactly to fp64 and
 * f and ⊕ are evaluated in fp64 (build: -O2 -fno-fast-math -ffp-contract=off);
 * int32 + and * wrap mod 2^32 (two's complement); PRL per reading C-18/C-19.
 *
 * Parallelism: OpenMP over the outermost cc dimension only; each output element is
 * computed by exactly one thread in the literal order, so results do not depend on
 * the thread count.  A spec without cc dimensions runs on one thread.
 *
 * Pins (tests/test_oracle_*.py, run with -m "not gpu"): math.fsum for fp32 dot,
 * closed forms mod 2^32 for int32 dot, A·I = A and ones·ones = K for MatMul, numpy
 * einsum / matmul in fp64, torch conv2d(stride=2) fp64, numpy slicing + constant /
 * linear-field closed forms for Jacobi, brute force + golden values for PRL, the
 * homomorphism split invariant, and brute-force operator algebra.
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <stdarg.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define O_MAXD 10
#define O_MAXR 8
#define O_MAXA 32  /* accesses per buffer (Gaussian_2D: 25 to one image, reading C-31) */
#define O_MAXX 40  /* input accesses in total (leaf gather array)                     */
#define O_MAXB 32
#define O_MAGIC 0x4D44484FLL /* 'MDHO' */

/* the oracle's own codes (independent of include/mdh.h) */
enum { T_BF16 = 0, T_F32 = 1, T_F64 = 2, T_I32 = 3, T_U32 = 4, T_I64 = 5 };
enum { C_CC = 0, C_ADD = 1, C_MAX = 2, C_MIN = 3, C_PRL_ARGMAX = 4, C_PRL_PAPER = 5, C_PS_ADD = 6 };
enum { S_MUL = 0, S_STENCIL = 1, S_PRL = 2, S_IDENTITY = 3 };
enum { K_FLOAT = 0, K_I32 = 1, K_U32 = 2, K_I64 = 3, K_PRL = 4 };

typedef struct {
  int dtype, rank, nacc;
  int64_t shape[O_MAXR];
  int64_t coeff[O_MAXA][O_MAXR][O_MAXD];
  int64_t off[O_MAXA][O_MAXR];
} obuf;

typedef struct {
  int D, f, nin, nout, nfp, kind;
  int64_t size[O_MAXD];
  int op[O_MAXD];
  const double* fp;
  obuf b[O_MAXB];          /* inputs then outputs */
  int ncc, nred;
  int cc[O_MAXD], red[O_MAXD];
} ospec;

/* one value of the tuple y(i): fp64 for floats, int64 for integers */
typedef struct { double f[3]; int64_t i[3]; } otuple;

static void seterr(char* err, int cap, const char* fmt, ...) {
  if (!err || cap <= 0) return;
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(err, (size_t)cap, fmt, ap);
  va_end(ap);
}

/* ---------------------------------------------------------------- spec decoding */
static int decode(const int64_t* e, int64_t n, const double* fp, int nfp, ospec* s,
                  char* err, int cap) {
  int64_t p = 0;
#define NEXT() (p < n ? e[p++] : (seterr(err, cap, "truncated spec"), (int64_t)-999999))
  memset(s, 0, sizeof(*s));
  if (NEXT() != O_MAGIC) { seterr(err, cap, "bad magic"); return -1; }
  s->D = (int)NEXT();
  if (s->D < 1 || s->D > O_MAXD) { seterr(err, cap, "bad D"); return -1; }
  for (int d = 0; d < s->D; ++d) s->size[d] = NEXT();
  for (int d = 0; d < s->D; ++d) s->op[d] = (int)NEXT();
  s->f = (int)NEXT();
  s->nin = (int)NEXT();
  s->nout = (int)NEXT();
  if (s->nin < 1 || s->nout < 1 || s->nin + s->nout > O_MAXB) { seterr(err, cap, "bad buffer count"); return -1; }
  for (int b = 0; b < s->nin + s->nout; ++b) {
    obuf* B = &s->b[b];
    B->dtype = (int)NEXT();
    B->rank = (int)NEXT();
    if (B->rank < 1 || B->rank > O_MAXR) { seterr(err, cap, "bad rank"); return -1; }
    for (int r = 0; r < B->rank; ++r) B->shape[r] = NEXT();
    B->nacc = (int)NEXT();
    if (B->nacc < 1 || B->nacc > O_MAXA) { seterr(err, cap, "bad access count"); return -1; }
    for (int a = 0; a < B->nacc; ++a) {
      for (int r = 0; r < B->rank; ++r)
        for (int d = 0; d < s->D; ++d) B->coeff[a][r][d] = NEXT();
      for (int r = 0; r < B->rank; ++r) B->off[a][r] = NEXT();
    }
  }
  if (p != n) { seterr(err, cap, "trailing spec data"); return -1; }
#undef NEXT
  s->fp = fp;
  s->nfp = nfp;
  for (int d = 0; d < s->D; ++d) {
    if (s->size[d] < 1) { seterr(err, cap, "size of dim %d < 1 (reading C-10)", d); return -1; }
    /* cc and ps dims are kept in the result; pw and ps dims are folded */
    if (s->op[d] == C_CC || s->op[d] == C_PS_ADD) s->cc[s->ncc++] = d;
    if (s->op[d] != C_CC) s->red[s->nred++] = d;
  }
  return 0;
}

static int is_float_t(int t) { return t == T_BF16 || t == T_F32 || t == T_F64; }

/* ------------------------------------------------- shapes and bound validation */
/* Range of coordinate r of access a over the index space; collapsed dims (pw)
 * are 0 for outputs (reading C-4). */
static void coord_range(const ospec* s, const obuf* B, int a, int r, int is_out,
                        int64_t* lo, int64_t* hi) {
  int64_t l = B->off[a][r], h = B->off[a][r];
  for (int d = 0; d < s->D; ++d) {
    int64_t ext = (is_out && s->op[d] != C_CC && s->op[d] != C_PS_ADD) ? 0 : s->size[d] - 1;
    int64_t c = B->coeff[a][r][d];
    if (c > 0) h += c * ext; else l += c * ext;
  }
  *lo = l; *hi = h;
}

static int finalize_shapes(ospec* s, char* err, int cap) {
  for (int b = 0; b < s->nin + s->nout; ++b) {
    obuf* B = &s->b[b];
    int is_out = b >= s->nin;
    int declared = 0;
    for (int r = 0; r < B->rank; ++r) declared |= (B->shape[r] != 0);
    for (int r = 0; r < B->rank; ++r) {
      int64_t mx = -1;
      for (int a = 0; a < B->nacc; ++a) {
        int64_t lo, hi;
        coord_range(s, B, a, r, is_out, &lo, &hi);
        if (lo < 0) { seterr(err, cap, "buffer %d access %d coord %d negative", b, a, r); return -1; }
        if (hi > mx) mx = hi;
      }
      if (declared) {   /* fn.7 P:316 / Listing 12: declared must contain accesses */
        if (B->shape[r] <= mx) { seterr(err, cap, "buffer %d declared shape too small", b); return -1; }
      } else {
        B->shape[r] = mx + 1;   /* reading C-9 */
      }
    }
  }
  return 0;
}

static int64_t buf_elems(const obuf* B) {
  int64_t n = 1;
  for (int r = 0; r < B->rank; ++r) n *= B->shape[r];
  return n;
}

/* row-major linear element index of access a at point idx (Listing 1 P:91 layout) */
static int64_t lin_index(const ospec* s, const obuf* B, int a, const int64_t* idx) {
  int64_t lin = 0;
  for (int r = 0; r < B->rank; ++r) {
    int64_t c = B->off[a][r];
    for (int d = 0; d < s->D; ++d) c += B->coeff[a][r][d] * idx[d];
    lin = lin * B->shape[r] + c;
  }
  return lin;
}

/* --------------------------------------------------------------- element access */
static double load_f(const void* p, int t, int64_t k) {
  switch (t) {
    case T_F32: return (double)((const float*)p)[k];
    case T_F64: return ((const double*)p)[k];
    case T_BF16: {
      uint32_t bits = ((uint32_t)((const uint16_t*)p)[k]) << 16;
      float f;
      memcpy(&f, &bits, 4);
      return (double)f;
    }
  }
  return 0.0;
}

static int64_t load_i(const void* p, int t, int64_t k) {
  switch (t) {
    case T_I32: return (int64_t)((const int32_t*)p)[k];
    case T_U32: return (int64_t)((const uint32_t*)p)[k];
    case T_I64: return ((const int64_t*)p)[k];
  }
  return 0;
}

static int64_t wrap(int kind, int64_t v) {
  if (kind == K_I32) return (int64_t)(int32_t)(uint32_t)(uint64_t)v;   /* mod 2^32, C-12 */
  if (kind == K_U32) return (int64_t)(uint32_t)(uint64_t)v;
  return v;                                                           /* i64: mod 2^64 */
}

/* ------------------------------------------------------------ catalog: f (SF) */
/* Leaf: y(i) = f(x(i)), x gathered through every input access in (b, a) order. */
static void leaf(const ospec* s, const void* const* in, const int64_t* idx, otuple* y) {
  double xf[O_MAXX] = {0};
  int64_t xi[O_MAXX] = {0};
  int n = 0;
  for (int b = 0; b < s->nin; ++b) {
    const obuf* B = &s->b[b];
    for (int a = 0; a < B->nacc; ++a) {
      int64_t k = lin_index(s, B, a, idx);
      if (is_float_t(B->dtype)) xf[n] = load_f(in[b], B->dtype, k);
      else xi[n] = load_i(in[b], B->dtype, k);
      ++n;
    }
  }
  switch (s->f) {
    case S_MUL:   /* f_mul */
      if (s->kind == K_FLOAT) y->f[0] = xf[0] * xf[1];
      else y->i[0] = wrap(s->kind, (int64_t)((uint64_t)xi[0] * (uint64_t)xi[1]));
      break;
    case S_IDENTITY:
      if (s->kind == K_FLOAT) y->f[0] = xf[0]; else y->i[0] = xi[0];
      break;
    case S_STENCIL: { /* Σ_a w_a x_a in access order, fp64 (reading C-16) */
      double acc = s->fp[0] * xf[0];
      for (int a = 1; a < n; ++a) acc = acc + s->fp[a] * xf[a];
      y->f[0] = acc;
      break;
    }
    case S_PRL: {     /* reading C-18: new_f0..7, db_f0..7, db_id */
      unsigned mask = 0;
      for (int k = 0; k < 8; ++k)
        if ((uint32_t)xi[k] == (uint32_t)xi[8 + k]) mask |= 1u << k;
      double w = 0.0;
      for (int k = 0; k < 8; ++k) w = w + ((mask >> k) & 1u ? s->fp[k] : s->fp[8 + k]);
      int pc = 0;
      for (int k = 0; k < 8; ++k) pc += (mask >> k) & 1u;
      y->i[0] = xi[16];                      /* match_id = db_id[i]  (Listing 11 l.35) */
      y->f[1] = w;                           /* match_weight                           */
      y->i[2] = (mask == 0xFFu) ? 14 : pc;   /* id_measure                             */
      break;
    }
  }
}

/* ---------------------------------------------------- catalog: ⊕ of pw(⊕) */
static void combine(const ospec* s, int op, const otuple* l, const otuple* r, otuple* res) {
  int nc = (s->f == S_PRL) ? 3 : 1;
  switch (op) {
    case C_ADD:
    case C_PS_ADD:
      for (int c = 0; c < nc; ++c) {
        if (s->kind == K_FLOAT) res->f[c] = l->f[c] + r->f[c];
        else res->i[c] = wrap(s->kind, (int64_t)((uint64_t)l->i[c] + (uint64_t)r->i[c]));
      }
      break;
    case C_MAX:
      for (int c = 0; c < nc; ++c) {
        if (s->kind == K_FLOAT) res->f[c] = (r->f[c] > l->f[c]) ? r->f[c] : l->f[c];
        else res->i[c] = (r->i[c] > l->i[c]) ? r->i[c] : l->i[c];
      }
      break;
    case C_MIN:
      for (int c = 0; c < nc; ++c) {
        if (s->kind == K_FLOAT) res->f[c] = (r->f[c] < l->f[c]) ? r->f[c] : l->f[c];
        else res->i[c] = (r->i[c] < l->i[c]) ? r->i[c] : l->i[c];
      }
      break;
    case C_PRL_ARGMAX: {   /* reading C-19: lexicographic max of (id==14, weight, match_id) */
      int l14 = l->i[2] == 14, r14 = r->i[2] == 14;
      int take_r;
      if (r14 != l14) take_r = r14 > l14;
      else if (r->f[1] != l->f[1]) take_r = r->f[1] > l->f[1];
      else take_r = r->i[0] > l->i[0];
      *res = take_r ? *r : *l;
      break;
    }
    case C_PRL_PAPER:      /* Listing 11 prl_max, literally */
      if (l->i[2] == 14 && r->i[2] != 14) *res = *l; else *res = *r;
      break;
  }
}

/* FOLD(t, idx): reduce the non-cc dims red[t..].  A pw dim folds its
 * whole range and collapses to index 0; a ps dim (prefix sum, Listing 17) keeps its index:
 * the result at output index k is the fold over [0, k] (inclusive; for a contiguous split
 * P|Q, res[q] = cf(lhs[max P], rhs[q]) with the lower index range as lhs, reading C-25). */
static void fold(const ospec* s, const void* const* in, int64_t* idx, const int64_t* keep, int t, otuple* out) {
  if (t == s->nred) { leaf(s, in, idx, out); return; }
  int d = s->red[t];
  int64_t last = s->op[d] == C_PS_ADD ? keep[d] : s->size[d] - 1;
  otuple acc, nxt, tmp;
  idx[d] = 0;
  fold(s, in, idx, keep, t + 1, &acc);
  for (int64_t v = 1; v <= last; ++v) {
    idx[d] = v;
    fold(s, in, idx, keep, t + 1, &nxt);
    combine(s, s->op[d], &acc, &nxt, &tmp);   /* lhs = lower index range */
    acc = tmp;
  }
  idx[d] = s->op[d] == C_PS_ADD ? keep[d] : 0;   /* output index: ps kept, pw collapsed (C-4) */
  *out = acc;
}

static void store(const ospec* s, void* const* out, const int64_t* idx, const otuple* y,
                  unsigned char* const* mark, int* collide) {
  int comp = 0;
  for (int b = 0; b < s->nout; ++b) {
    const obuf* B = &s->b[s->nin + b];
    for (int a = 0; a < B->nacc; ++a, ++comp) {
      int64_t k = lin_index(s, B, a, idx);   /* idx has pw dims = 0 (reading C-4) */
      if (mark) {
        if (__atomic_exchange_n(&mark[b][k], (unsigned char)1, __ATOMIC_RELAXED)) *collide = 1;
      }
      int c = (s->f == S_PRL) ? b : 0;
      switch (B->dtype) {
        case T_F32: case T_BF16: case T_F64: ((double*)out[b])[k] = y->f[c]; break;   /* fp64 result */
        case T_I32: ((int32_t*)out[b])[k] = (int32_t)y->i[c]; break;
        case T_U32: ((uint32_t*)out[b])[k] = (uint32_t)y->i[c]; break;
        case T_I64: ((int64_t*)out[b])[k] = y->i[c]; break;
      }
    }
  }
}

static int check_catalog(ospec* s, char* err, int cap) {
  int nacc = 0, allf = 1, alli = 1, t0 = s->b[0].dtype;
  for (int b = 0; b < s->nin; ++b) {
    nacc += s->b[b].nacc;
    if (is_float_t(s->b[b].dtype)) alli = 0; else allf = 0;
  }
  int nout_acc = 0;
  for (int b = 0; b < s->nout; ++b) nout_acc += s->b[s->nin + b].nacc;
  if (nacc > O_MAXX) { seterr(err, cap, "more than 40 input accesses"); return -1; }
  int redop = -1;
  for (int t = 0; t < s->nred; ++t) {
    if (redop >= 0 && s->op[s->red[t]] != redop) { /* reading C-3: evaluated anyway */ }
    redop = s->op[s->red[t]];
  }
  if (s->f == S_PRL) {
    if (nacc != 17 || s->nout != 3 || s->nfp != 16) { seterr(err, cap, "PRL arity"); return -1; }
    s->kind = K_PRL;
    for (int t = 0; t < s->nred; ++t)
      if (s->op[s->red[t]] != C_PRL_ARGMAX && s->op[s->red[t]] != C_PRL_PAPER) { seterr(err, cap, "PRL op"); return -1; }
    return 0;
  }
  for (int t = 0; t < s->nred; ++t)
    if (s->op[s->red[t]] == C_PRL_ARGMAX || s->op[s->red[t]] == C_PRL_PAPER) { seterr(err, cap, "PRL op on scalar f"); return -1; }
  if (nout_acc != 1) { seterr(err, cap, "scalar f needs exactly one output access"); return -1; }
  if (s->f == S_MUL && nacc != 2) { seterr(err, cap, "MUL arity"); return -1; }
  if (s->f == S_IDENTITY && nacc != 1) { seterr(err, cap, "IDENTITY arity"); return -1; }
  if (s->f == S_STENCIL && (nacc != s->nfp || !allf)) { seterr(err, cap, "STENCIL arity"); return -1; }
  if (allf) s->kind = K_FLOAT;
  else if (alli) s->kind = (t0 == T_I64) ? K_I64 : (t0 == T_U32 ? K_U32 : K_I32);
  else { seterr(err, cap, "mixed int/float inputs"); return -1; }
  int ot = s->b[s->nin].dtype;
  if (s->kind == K_FLOAT && !is_float_t(ot)) { seterr(err, cap, "float f into int output"); return -1; }
  if (s->kind != K_FLOAT && is_float_t(ot)) { seterr(err, cap, "int f into float output"); return -1; }
  return 0;
}

static int prepare(const int64_t* enc, int64_t n, const double* fp, int nfp, ospec* s,
                   char* err, int cap) {
  if (decode(enc, n, fp, nfp, s, err, cap)) return -1;
  if (check_catalog(s, err, cap)) return -1;
  if (finalize_shapes(s, err, cap)) return -1;
  return 0;
}

/* ------------------------------------------------------------------ exports */

/* Shapes (declared or inferred) of all buffers: out[(b)*8 + r]. */
int mdho_shapes(const int64_t* enc, int64_t n, const double* fp, int nfp, int64_t* shapes,
                char* err, int cap) {
  ospec* sp = (ospec*)calloc(1, sizeof(ospec));   /* ~0.7 MB: heap, not stack */
  if (!sp) { seterr(err, cap, "oom"); return -1; }
  if (prepare(enc, n, fp, nfp, sp, err, cap)) { free(sp); return -1; }
  for (int b = 0; b < sp->nin + sp->nout; ++b)
    for (int r = 0; r < O_MAXR; ++r) shapes[b * O_MAXR + r] = r < sp->b[b].rank ? sp->b[b].shape[r] : 0;
  { free(sp); return 0; }
}

/* Full evaluation.  Float outputs are written as fp64 arrays; integer outputs in
 * their own type.  Elements outside the image of ω are untouched (reading C-5). */
int mdho_eval(const int64_t* enc, int64_t n, const double* fp, int nfp,
              const void* const* in, void* const* out, int nthreads, char* err, int cap) {
  ospec* sp = (ospec*)calloc(1, sizeof(ospec));   /* ~0.7 MB: heap, not stack */
  if (!sp) { seterr(err, cap, "oom"); return -1; }
  if (prepare(enc, n, fp, nfp, sp, err, cap)) { free(sp); return -1; }
  unsigned char* mark[O_MAXB];
  for (int b = 0; b < sp->nout; ++b) {
    mark[b] = (unsigned char*)calloc((size_t)buf_elems(&sp->b[sp->nin + b]), 1);
    if (!mark[b]) { seterr(err, cap, "oom"); { free(sp); return -1; } }
  }
  int collide = 0;
  int64_t outer = sp->ncc > 0 ? sp->size[sp->cc[0]] : 1;
  int64_t inner = 1;
  for (int t = 1; t < sp->ncc; ++t) inner *= sp->size[sp->cc[t]];
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#pragma omp parallel for schedule(dynamic, 1) if (sp->ncc > 0)
#endif
  for (int64_t o = 0; o < outer; ++o) {
    int64_t idx[O_MAXD];
    otuple y;
    memset(idx, 0, sizeof(idx));
    for (int64_t q = 0; q < inner; ++q) {
      /* cc coordinate j in lexicographic (dimension) order */
      int64_t rem = q;
      for (int t = sp->ncc - 1; t >= 1; --t) {
        idx[sp->cc[t]] = rem % sp->size[sp->cc[t]];
        rem /= sp->size[sp->cc[t]];
      }
      if (sp->ncc > 0) idx[sp->cc[0]] = o;
      memset(&y, 0, sizeof(y));
      int64_t keep[O_MAXD];
      memcpy(keep, idx, sizeof(keep));
      fold(sp, in, idx, keep, 0, &y);
      store(sp, out, idx, &y, mark, &collide);
    }
  }
  for (int b = 0; b < sp->nout; ++b) free(mark[b]);
  if (collide) { seterr(err, cap, "output index function not injective (reading C-5)"); { free(sp); return -2; } }
  { free(sp); return 0; }
}

/* Sampled evaluation at n_points cc coordinates (points: n_points × D full
 * coordinates; pw entries ignored).  For every output buffer b (its access 0) and
 * point p: lin[b*np+p] = linear element index, vf/vi[b*np+p] = the value (float
 * outputs in vf as fp64, integer outputs in vi).                               */
int mdho_eval_points(const int64_t* enc, int64_t n, const double* fp, int nfp,
                     const void* const* in, int64_t np, const int64_t* points,
                     int64_t* lin, double* vf, int64_t* vi, int nthreads, char* err, int cap) {
  ospec* sp = (ospec*)calloc(1, sizeof(ospec));   /* ~0.7 MB: heap, not stack */
  if (!sp) { seterr(err, cap, "oom"); return -1; }
  if (prepare(enc, n, fp, nfp, sp, err, cap)) { free(sp); return -1; }
  for (int64_t p = 0; p < np; ++p)
    for (int t = 0; t < sp->ncc; ++t) {
      int64_t v = points[p * sp->D + sp->cc[t]];
      if (v < 0 || v >= sp->size[sp->cc[t]]) { seterr(err, cap, "point out of range"); { free(sp); return -1; } }
    }
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#pragma omp parallel for schedule(dynamic, 16)
#endif
  for (int64_t p = 0; p < np; ++p) {
    int64_t idx[O_MAXD];
    otuple y;
    memset(idx, 0, sizeof(idx));
    for (int t = 0; t < sp->ncc; ++t) idx[sp->cc[t]] = points[p * sp->D + sp->cc[t]];
    memset(&y, 0, sizeof(y));
    int64_t keep[O_MAXD];
    memcpy(keep, idx, sizeof(keep));
    fold(sp, in, idx, keep, 0, &y);
    for (int b = 0; b < sp->nout; ++b) {
      const obuf* B = &sp->b[sp->nin + b];
      int c = (sp->f == S_PRL) ? b : 0;
      lin[b * np + p] = lin_index(sp, B, 0, idx);
      if (is_float_t(B->dtype)) vf[b * np + p] = y.f[c];
      else vi[b * np + p] = y.i[c];
    }
  }
  { free(sp); return 0; }
}

/* Ordered ⊗-fold of two partial results given as tuples (used by the homomorphism
 * tests to recombine split evaluations exactly as Listing 16 does). kind: see enum.
 * lf/li, rf/ri: per component (3) fp64 / int64.  Writes the result into lf/li.   */
int mdho_combine_tuple(int op, int f, int kind, double* lf, int64_t* li, const double* rf,
                       const int64_t* ri) {
  static __thread ospec* sp = NULL;     /* combine() reads only f and kind */
  if (!sp && !(sp = (ospec*)calloc(1, sizeof(ospec)))) return -1;
  sp->f = f;
  sp->kind = kind;
  otuple l, r, res;
  for (int c = 0; c < 3; ++c) { l.f[c] = lf[c]; l.i[c] = li[c]; r.f[c] = rf[c]; r.i[c] = ri[c]; }
  res = l;
  combine(sp, op, &l, &r, &res);
  for (int c = 0; c < 3; ++c) { lf[c] = res.f[c]; li[c] = res.i[c]; }
  return 0;
}

int mdho_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
