// tiles.cpp — the tile selector (north-star subsystem 3).
//
// Template parameters come from a table produced by a MEASURED sweep on B200
// (tools/sweep_tiles.py → tiles/b200.json; the ATF auto-tuning of P:497-501 is prior
// art, replaced by this sweep).  Key: (template, dtype, f, ⊗-class, shape bucket), the
// bucket being the log2-rounded extents of (Ncc, Nred) or (M, N, K) of THIS rank's
// sub-problem; f ("MUL", "STENCIL", "PRL_COMPARE", "IDENTITY") and the ⊗-class (the
// common pw operator: "PW_ADD", …, "PS_ADD", or "CC") must match when an entry records
// them (entries without them match any f / ⊗).
// Lookup: exact bucket, else the nearest bucket of the same template and dtype by
// log-distance, else the template's defaults.  Overrides: the plan option force_tile or
// $MDH_FORCE_TILE ("split=4,zchunk=16,…").  Table: the plan option, $MDH_TILE_TABLE, or
// the copy compiled into the library at build time.
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <map>
#include <memory>
#include <sstream>
#include <string>
#include <vector>

#include "internal.h"

namespace mdh {

static const char* kBuiltinTable =
#include "tiles_builtin.inc"
    ;

namespace {
// ---- a minimal JSON reader (objects, arrays, strings, numbers, true/false/null) ----
struct J {
  enum T { NUL, NUM, STR, ARR, OBJ, BOOL } t = NUL;
  double num = 0;
  std::string str;
  std::vector<J> arr;
  std::vector<std::pair<std::string, J>> obj;
  const J* get(const char* k) const {
    for (auto& kv : obj)
      if (kv.first == k) return &kv.second;
    return nullptr;
  }
};

struct Parser {
  const char* s;
  bool ok = true;
  void ws() { while (*s == ' ' || *s == '\n' || *s == '\t' || *s == '\r') ++s; }
  std::string string() {
    std::string r;
    ++s;
    while (*s && *s != '"') {
      if (*s == '\\' && s[1]) ++s;
      r += *s++;
    }
    if (*s == '"') ++s; else ok = false;
    return r;
  }
  J value() {
    ws();
    J v;
    if (*s == '{') {
      v.t = J::OBJ;
      ++s;
      ws();
      if (*s == '}') { ++s; return v; }
      while (ok) {
        ws();
        if (*s != '"') { ok = false; break; }
        std::string k = string();
        ws();
        if (*s != ':') { ok = false; break; }
        ++s;
        v.obj.push_back({k, value()});
        ws();
        if (*s == ',') { ++s; continue; }
        if (*s == '}') { ++s; break; }
        ok = false;
      }
    } else if (*s == '[') {
      v.t = J::ARR;
      ++s;
      ws();
      if (*s == ']') { ++s; return v; }
      while (ok) {
        v.arr.push_back(value());
        ws();
        if (*s == ',') { ++s; continue; }
        if (*s == ']') { ++s; break; }
        ok = false;
      }
    } else if (*s == '"') {
      v.t = J::STR;
      v.str = string();
    } else if (!std::strncmp(s, "true", 4)) { v.t = J::BOOL; v.num = 1; s += 4; }
    else if (!std::strncmp(s, "false", 5)) { v.t = J::BOOL; s += 5; }
    else if (!std::strncmp(s, "null", 4)) { s += 4; }
    else {
      char* e = nullptr;
      v.t = J::NUM;
      v.num = std::strtod(s, &e);
      if (e == s) ok = false;
      s = e;
    }
    return v;
  }
};

const char* dtype_name(mdh_dtype t) {
  switch (t) {
    case MDH_BF16: return "bf16";
    case MDH_F32: return "f32";
    case MDH_F64: return "f64";
    case MDH_I32: return "i32";
    case MDH_U32: return "u32";
    case MDH_I64: return "i64";
  }
  return "?";
}

void shape_key(const Plan& p, double key[3]) {
  key[0] = key[1] = key[2] = 0;
  if (p.tmpl == T3_SIMT || p.tmpl == T4_TC) {
    key[0] = std::log2((double)p.con.M);
    key[1] = std::log2((double)p.con.N);
    key[2] = std::log2((double)p.con.K * (double)p.con.Z);
  } else {
    key[0] = std::log2((double)p.Ncc);
    key[1] = std::log2((double)p.Nred);
  }
}

const char* fn_name(mdh_fn f) {
  switch (f) {
    case MDH_F_MUL: return "MUL";
    case MDH_F_STENCIL: return "STENCIL";
    case MDH_F_PRL_COMPARE: return "PRL_COMPARE";
    case MDH_F_IDENTITY: return "IDENTITY";
  }
  return "?";
}

const char* op_class(const Plan& p) {
  if (p.nps > 0) return "PS_ADD";
  switch (p.redop) {
    case MDH_PW_ADD: return "PW_ADD";
    case MDH_PW_MAX: return "PW_MAX";
    case MDH_PW_MIN: return "PW_MIN";
    case MDH_PW_PRL_ARGMAX: return "PW_PRL_ARGMAX";
    case MDH_PW_PRL_PAPER: return "PW_PRL_PAPER";
    default: return "CC";
  }
}

void apply(Tiles* t, const std::string& k, double v) {
  int iv = (int)v;
  if (k == "threads") t->threads = iv;
  else if (k == "bm") t->bm = iv;
  else if (k == "bn") t->bn = iv;
  else if (k == "bk") t->bk = iv;
  else if (k == "split") t->split = iv;
  else if (k == "stages") t->stages = iv;
  else if (k == "vec") t->vec = iv;
  else if (k == "zchunk") t->zchunk = iv;
  else if (k == "seg") t->seg = iv;
  else if (k == "per_thread") t->per_thread = iv;
  else if (k == "cluster") t->cluster = iv;
  else if (k == "implicit") t->implicit = iv;
  else if (k == "epi") t->epi = iv;
  else if (k == "krot") t->krot = iv;
  else if (k == "l2pf") t->l2pf = iv;
  else if (k == "nstream") t->nstream = iv;
  else if (k == "areuse") t->areuse = iv;
  else if (k == "mode") t->mode = iv;
}

std::string read_file(const char* path) {
  std::ifstream f(path);
  if (!f) return "";
  std::stringstream ss;
  ss << f.rdbuf();
  return ss.str();
}
}  // namespace

void lookup_tiles(Plan* p, const char* table_path, const char* force) {
  Tiles t;
  // template defaults
  if (p->tmpl == T1_STENCIL) { t.zchunk = 32; t.stages = 0; }   // stages ≥ 3: TMA-staged 7-point kernel
  // T4: bn, cluster, stages 0 = auto (stages = 4 selects the 4-stage wide 2-SM ring)
  if (p->tmpl == T4_TC) { t.bm = 128; t.bn = 0; t.bk = 64; t.stages = 0; t.cluster = 0; }
  // T5: 4 new records per thread, registers for 3 CTAs per SM, DB loop unrolled ×4 (t5_prl.cu)
  if (p->tmpl == T5_PRL) { t.vec = 4; t.stages = 3; t.bk = 4; }
  std::string text;
  const char* path = table_path ? table_path : std::getenv("MDH_TILE_TABLE");
  if (path && *path) text = read_file(path);
  if (text.empty()) text = kBuiltinTable;
  Parser ps{text.c_str()};
  J root = ps.value();
  const J* entries = ps.ok ? root.get("entries") : nullptr;
  double key[3];
  shape_key(*p, key);
  const char* tname = template_name(p->tmpl);
  mdh_dtype dt = p->n_in > 0 ? p->in[0].dtype : MDH_F32;
  const char* dname = dtype_name(dt);
  const J* best = nullptr;
  double bestd = 1e30;
  if (entries && entries->t == J::ARR) {
    for (const J& e : entries->arr) {
      const J* et = e.get("template");
      const J* ed = e.get("dtype");
      const J* eb = e.get("bucket");
      if (!et || !ed || !eb || et->str != tname || ed->str != dname || eb->t != J::ARR) continue;
      const J* ef = e.get("f");
      const J* eo = e.get("op");
      if ((ef && ef->str != fn_name(p->f)) || (eo && eo->str != op_class(*p))) continue;
      double d = 0;
      for (size_t i = 0; i < eb->arr.size() && i < 3; ++i) d += std::fabs(eb->arr[i].num - key[i]);
      if (d < bestd) { bestd = d; best = &e; }
    }
  }
  // a measured entry more than 6 octaves (summed log2 distance) away says nothing about
  // this shape: keep the template defaults then
  if (best && bestd <= 6.0) {
    const J* tl = best->get("tiles");
    if (tl)
      for (auto& kv : tl->obj) apply(&t, kv.first, kv.second.num);
    char b[96];
    std::snprintf(b, sizeof(b), "table(dist=%.2f)", bestd);
    t.source = b;
  }
  const char* f = force ? force : std::getenv("MDH_FORCE_TILE");
  if (f && *f) {
    std::string s(f);
    size_t pos = 0;
    while (pos < s.size()) {
      size_t c = s.find(',', pos);
      std::string kv = s.substr(pos, c == std::string::npos ? std::string::npos : c - pos);
      size_t eq = kv.find('=');
      if (eq != std::string::npos) apply(&t, kv.substr(0, eq), std::atof(kv.c_str() + eq + 1));
      if (c == std::string::npos) break;
      pos = c + 1;
    }
    t.source += "+forced";
  }
  p->tiles = t;
}

}  // namespace mdh
