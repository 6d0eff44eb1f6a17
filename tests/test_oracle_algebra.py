"""Homomorphism split invariant and catalog-operator algebra of the oracle
(SURVEY §8(c).4 rows "Homomorphism invariant" and "Catalog operator algebra").

The split sub-specs and the recombination are written here, independently of both
the oracle and the CUDA partitioner: splitting dim d at s gives the sub-domains
[0,s) and [s,I_d) (the second one by shifting every access offset by coeff[:,d]*s);
a cc split concatenates by index (Listing 15), a pw split combines with ⊕ (Listing 16).
"""
import copy
import itertools

import numpy as np
import pytest

import oracle
from mdh_workloads import gen as G
from mdh_workloads import specs as S

INF = float("inf")


def split_spec(spec, d, s, shapes):
    lo, hi = copy.deepcopy(spec), copy.deepcopy(spec)
    lo["sizes"][d] = s
    hi["sizes"][d] = spec["sizes"][d] - s
    nin = len(spec["inputs"])
    for sub in (lo, hi):
        for b, buf in enumerate(sub["inputs"] + sub["outputs"]):
            buf["shape"] = list(shapes[b])
    for b, buf in enumerate(hi["inputs"] + hi["outputs"]):
        if b >= nin and spec["ops"][d] != "CC":
            continue                     # collapsed pw index stays 0 (reading C-4)
        for acc in buf["acc"]:
            for r in range(len(acc["offset"])):
                acc["offset"][r] += acc["coeff"][r][d] * s
    return lo, hi


def py_combine(op, l, r):
    """⊕ written independently (Listing 16 with cf; readings C-12, C-19)."""
    if op == "PW_ADD":
        return l + r
    if op == "PW_MAX":
        return np.maximum(l, r)
    if op == "PW_MIN":
        return np.minimum(l, r)
    raise ValueError(op)


def prl_combine(op, l, r):
    (li, lw, lm), (ri, rw, rm) = l, r
    if op == "PW_PRL_PAPER":
        take_l = (lm == 14) & (rm != 14)
    else:
        kl = np.stack([(lm == 14).astype(np.float64), lw, li.astype(np.float64)])
        kr = np.stack([(rm == 14).astype(np.float64), rw, ri.astype(np.float64)])
        take_l = np.ones(li.shape, bool)
        decided = np.zeros(li.shape, bool)
        for c in range(3):
            gt = (kr[c] > kl[c]) & ~decided
            lt = (kr[c] < kl[c]) & ~decided
            take_l[gt] = False
            decided |= gt | lt
        # exact ties keep lhs (identical records)
    return (np.where(take_l, li, ri), np.where(take_l, lw, rw), np.where(take_l, lm, rm))


CASES = [
    ("dot_f32", lambda: S.dot(1000, "f32"), lambda sp: G.dot_inputs(1000, "f32")),
    ("dot_i32", lambda: S.dot(1000, "i32"), lambda sp: G.dot_inputs(1000, "i32")),
    ("dot_max", lambda: S.dot(777, "f32", "PW_MAX"), lambda sp: G.dot_inputs(777, "f32")),
    ("matvec_min", lambda: S.matvec(9, 50, "i32", "PW_MIN"), lambda sp: G.gen_inputs(sp, 10)),
    ("matmul", lambda: S.matmul(6, 7, 30), lambda sp: G.matmul_inputs(6, 7, 30)),
    ("jacobi3d", lambda: S.jacobi3d(6, 7, 8), lambda sp: G.jacobi3d_inputs(6, 7, 8)),
    ("mcc", lambda: S.mcc(2, 3, 3, 4, 3, 3, 2, "f32"), lambda sp: G.mcc_inputs(sp)),
    ("ccsd", lambda: S.ccsd_sd1(2, 3, "f32"), lambda sp: G.gen_inputs(sp, 40)),
]


@pytest.mark.parametrize("name,mk,mkin", CASES, ids=[c[0] for c in CASES])
def test_homomorphism_split_every_dim(name, mk, mkin):
    spec = mk()
    ins = mkin(spec)
    shapes = oracle.shapes(spec)
    full = oracle.evaluate(spec, ins)
    g = np.random.Generator(np.random.PCG64(123))
    for d in range(spec["D"]):
        if spec["sizes"][d] < 2:
            continue
        s = int(g.integers(1, spec["sizes"][d]))
        lo, hi = split_spec(spec, d, s, shapes)
        if spec["ops"][d] == "CC":
            a = oracle.evaluate(lo, ins, fill=np.nan)
            b = oracle.evaluate(hi, ins, fill=np.nan)
            for o, oa, ob in zip(full, a, b):
                if o.dtype.kind == "f":
                    merged = np.where(np.isnan(oa), ob, oa)
                else:
                    continue  # integer cc split covered by float cases
                assert np.array_equal(merged, o), (name, d)
        else:
            a = oracle.evaluate(lo, ins)
            b = oracle.evaluate(hi, ins)
            comb = py_combine(spec["ops"][d], a[0], b[0])
            if full[0].dtype.kind == "f" and spec["ops"][d] == "PW_ADD":
                scale = np.maximum(np.abs(full[0]), 1e-300)
                assert np.max(np.abs(comb - full[0]) / scale) < 1e-9, (name, d)
            elif full[0].dtype == np.int32:
                assert np.array_equal(comb.astype(np.int64).astype(np.uint32).view(np.int32)
                                      if comb.dtype != np.int32 else comb, full[0])
            else:
                assert np.array_equal(comb, full[0]), (name, d)


@pytest.mark.parametrize("op", ["PW_PRL_ARGMAX", "PW_PRL_PAPER"])
def test_homomorphism_prl(op):
    N, I = 40, 300
    ins = G.prl_inputs(N, I, seed_base=5400)
    ins = [(x % 2).astype(np.uint32) if 8 <= k < 16 or k < 8 else x for k, x in enumerate(ins)]
    spec = S.prl(N, I, op)
    shapes = oracle.shapes(spec)
    full = oracle.evaluate(spec, ins)
    for s in (1, 7, 150, 299):
        lo, hi = split_spec(spec, 1, s, shapes)
        a = oracle.evaluate(lo, ins)
        b = oracle.evaluate(hi, ins)
        comb = prl_combine(op, a, b)
        for c in range(3):
            assert np.array_equal(comb[c], full[c]), (op, s, c)


# ------------------------------------------------------------- operator algebra
def _prl_vals():
    """Records as the PRL f produces them: match_id identifies the DB record, so equal
    match_id implies an equal record; weights tie across different ids."""
    vals = []
    mid = 100
    for idm in (0, 7, 14):
        for w in (-1.0, 2.5):
            for _ in range(2):
                vals.append(((0.0, w, 0.0), (mid, 0, idm)))
                mid += 1
    return vals


def _op(op, l, r):
    lf, li = oracle.combine_tuple(op, "PRL_COMPARE", 4, l, r)
    return (tuple(lf.tolist()), tuple(li.tolist()))


@pytest.mark.parametrize("op", ["PW_PRL_ARGMAX", "PW_PRL_PAPER"])
def test_prl_operator_algebra(op):
    V = _prl_vals()
    for a, b, c in itertools.product(V, repeat=3):
        assert _op(op, _op(op, a, b), c) == _op(op, a, _op(op, b, c))     # associative (C-2)
    comm = all(_op(op, a, b) == _op(op, b, a) for a, b in itertools.product(V, repeat=2))
    if op == "PW_PRL_ARGMAX":
        assert comm
        e = ((0.0, -INF, 0.0), (-(1 << 63), 0, -1))                       # identity (C-11)
        for a in V:
            assert _op(op, e, a) == _op(op, a, e) == (tuple(map(float, a[0])), tuple(a[1]))
    else:
        assert not comm                                                    # Listing 11 rule
        e = ((0.0, 0.0, 0.0), (0, 0, 0))                                   # any id != 14
        for a in V:
            assert _op(op, e, a) == (tuple(map(float, a[0])), tuple(a[1]))  # left identity only


def test_paper_rule_strided_split_differs():
    """the literal rule is not commutative, so a strided (round-robin)
    2-way split of the reduction dim gives a different result than the in-order fold."""
    g = np.random.Generator(np.random.PCG64(5))
    diffs = 0
    for _ in range(300):
        seq = [((0.0, float(g.integers(0, 3)), 0.0), (int(i), 0, int(g.choice([0, 14]))))
               for i in range(6)]
        acc = seq[0]
        for x in seq[1:]:
            acc = _op("PW_PRL_PAPER", acc, x)
        ev, od = seq[0::2], seq[1::2]
        a = ev[0]
        for x in ev[1:]:
            a = _op("PW_PRL_PAPER", a, x)
        b = od[0]
        for x in od[1:]:
            b = _op("PW_PRL_PAPER", b, x)
        diffs += _op("PW_PRL_PAPER", a, b) != acc
    assert diffs > 0


@pytest.mark.parametrize("op", ["PW_ADD", "PW_MAX", "PW_MIN"])
def test_int32_ops_associative_commutative(op):
    vals = [-(1 << 31), -5, -1, 0, 1, 3, (1 << 31) - 1]

    def f(a, b):
        lf, li = oracle.combine_tuple(op, "MUL", 1, ((0, 0, 0), (a, 0, 0)), ((0, 0, 0), (b, 0, 0)))
        return int(li[0])
    for a, b, c in itertools.product(vals, repeat=3):
        assert f(f(a, b), c) == f(a, f(b, c))
        assert f(a, b) == f(b, a)
    assert f((1 << 31) - 1, 1) == (-(1 << 31) if op == "PW_ADD" else f(1, (1 << 31) - 1))


def test_mixed_operator_interchange_counterexample():
    """Reading C-3: mixing pw(max) and pw(add) breaks the interchange law, so the result
    depends on the nesting order; the oracle evaluates the formula's order (⊗_1 outer)."""
    d = ["a", "b"]
    sp = S.make_spec("mixed", d, [2, 2], ["PW_MAX", "PW_ADD"], "IDENTITY",
                     [S.buffer("x", "f32", [["a", "b"]], d)], [S.buffer("y", "f32", [["0"]], d, shape=[1])])
    x = np.array([[1, 4], [5, 0]], np.float32)          # y[a,b]
    r = oracle.evaluate(sp, [x])[0][0]
    assert r == max(1 + 4, 5 + 0) == 5                   # max_a Σ_b y
    assert max(1, 5) + max(4, 0) == 9                    # the other order
