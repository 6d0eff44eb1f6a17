// prl_common.cuh — the PRL record and its two custom pw operators (device side).
//   PW_PRL_ARGMAX (reading C-19): keep the lexicographically larger (id==14, weight,
//     match_id); associative and commutative; exact ties are identical records.
//   PW_PRL_PAPER  (Listing 11 prl_max): res = lhs if lhs.id==14 and
//     rhs.id!=14 else rhs; associative, NOT commutative, so every GPU combine passes
//     (lower index range, higher index range) as (lhs, rhs) (reading C-2).
#pragma once
#include <stdint.h>

#include "../../include/mdh.h"

namespace mdh {

struct PrlRec {
  long long id;   // match_id
  double w;       // match_weight
  int m;          // id_measure
};

__device__ __forceinline__ bool prl_argmax_takes_rhs(const PrlRec& l, const PrlRec& r) {
  bool l14 = l.m == 14, r14 = r.m == 14;
  if (l14 != r14) return r14;
  if (r.w != l.w) return r.w > l.w;
  return r.id > l.id;
}

__device__ __forceinline__ PrlRec prl_combine(int op, const PrlRec& l, const PrlRec& r) {
  if (op == MDH_PW_PRL_PAPER) return (l.m == 14 && r.m != 14) ? l : r;
  return prl_argmax_takes_rhs(l, r) ? r : l;
}

}  // namespace mdh
