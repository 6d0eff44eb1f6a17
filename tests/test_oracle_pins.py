"""Pins of the CPU oracle against things other than itself.

Every check compares the oracle's literal loop nest with a closed form, a library
routine (math.fsum, numpy, torch CPU fp64), a brute-force evaluation written here,
or a golden value under tests/golden/ (each with its citation).  CPU only.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
from mdh_workloads import gen as G
from mdh_workloads import specs as S

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def f64(x, dt="f32"):
    if dt == "bf16":
        return G.bf16_bits_to_f32(x).astype(np.float64)
    return np.asarray(x, np.float64)


# ------------------------------------------------------------------ Dot (C1)
@pytest.mark.parametrize("kind", ["signed", "positive"])
def test_dot_fp32_vs_fsum(kind):
    """fp32×fp32 products are exact in fp64, so math.fsum gives the correctly rounded
    exact dot; the literal sequential fp64 fold must agree to ≤1e-12 relative."""
    N = 1 << 20
    x = G.dot_inputs(N, "f32", kind)
    r = oracle.evaluate(S.dot(N, "f32"), x)[0][0]
    exact = math.fsum((x[0].astype(np.float64) * x[1].astype(np.float64)).tolist())
    assert abs(r - exact) <= 1e-12 * abs(exact)


def test_dot_int32_closed_forms():
    g = gold("dot_int32.json")
    N = g["N"]
    # closed forms, evaluated with Python big ints, then mod 2^32 as int32 (reading C-12)
    def as_i32(v):
        v &= 0xFFFFFFFF
        return v - (1 << 32) if v >= (1 << 31) else v
    assert as_i32(N * (N - 1) // 2) == g["iota_one"]
    assert as_i32(N * (N - 1) * (2 * N - 1) // 6) == g["iota_iota"]
    sp = S.dot(N, "i32")
    assert oracle.evaluate(sp, G.dot_inputs(N, "i32", "iota_one"))[0][0] == g["iota_one"]
    assert oracle.evaluate(sp, G.dot_inputs(N, "i32", "iota_iota"))[0][0] == g["iota_iota"]


def test_dot_int32_random_wraps():
    N = 1 << 18
    a, b = G.dot_inputs(N, "i32")
    r = oracle.evaluate(S.dot(N, "i32"), [a, b])[0][0]
    true = int((a.astype(np.int64) * b.astype(np.int64)).sum())
    v = true & 0xFFFFFFFF
    assert r == (v - (1 << 32) if v >= 1 << 31 else v)


@pytest.mark.parametrize("op,fn", [("PW_MAX", np.max), ("PW_MIN", np.min)])
@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_dot_maxmin(op, fn, dt):
    N = 4097
    a, b = G.dot_inputs(N, dt)
    r = oracle.evaluate(S.dot(N, dt, op), [a, b])[0][0]
    if dt == "f32":
        assert r == fn(a.astype(np.float64) * b.astype(np.float64))
    else:
        prod = (a.astype(np.int64) * b.astype(np.int64)) & 0xFFFFFFFF
        prod = np.where(prod >= 1 << 31, prod - (1 << 32), prod)
        assert r == fn(prod)


# --------------------------------------------------------------- MatMul (C2)
def test_u32_and_i64_wrap_branches():
    """The oracle's uint32 (mod 2^32, unsigned order) and int64 (mod 2^64) kinds against
    Python's unbounded integers reduced by hand — independent of numpy's own wrapping."""
    g = np.random.Generator(np.random.PCG64(61))
    n = 3001
    a = g.integers(0, 2 ** 32, n, dtype=np.uint64).astype(np.uint32)
    b = g.integers(0, 2 ** 32, n, dtype=np.uint64).astype(np.uint32)
    exact = sum(int(x) * int(y) for x, y in zip(a.tolist(), b.tolist()))
    got = int(oracle.evaluate(S.dot(n, "u32"), [a, b])[0][0])
    assert got == exact % 2 ** 32
    # unsigned order: products ≥ 2^31 must win a max / lose a min as unsigned values
    prods = [(int(x) * int(y)) % 2 ** 32 for x, y in zip(a.tolist(), b.tolist())]
    assert int(oracle.evaluate(S.dot(n, "u32", "PW_MAX"), [a, b])[0][0]) == max(prods)
    assert int(oracle.evaluate(S.dot(n, "u32", "PW_MIN"), [a, b])[0][0]) == min(prods)
    # int64: products of ~2^40 × ~2^30 overflow 2^63; the sum wraps mod 2^64 (two's complement)
    x = (g.integers(-2 ** 40, 2 ** 40, n)).astype(np.int64)
    y = (g.integers(-2 ** 30, 2 ** 30, n)).astype(np.int64)
    exact = sum(int(p) * int(q) for p, q in zip(x.tolist(), y.tolist())) % 2 ** 64
    exact = exact - 2 ** 64 if exact >= 2 ** 63 else exact
    assert int(oracle.evaluate(S.dot(n, "i64"), [x, y])[0][0]) == exact
    prods64 = [int(p) * int(q) for p, q in zip(x.tolist(), y.tolist())]
    wrap64 = [((v + 2 ** 63) % 2 ** 64) - 2 ** 63 for v in prods64]
    assert int(oracle.evaluate(S.dot(n, "i64", "PW_MAX"), [x, y])[0][0]) == max(wrap64)
    assert int(oracle.evaluate(S.dot(n, "i64", "PW_MIN"), [x, y])[0][0]) == min(wrap64)


def test_matmul_identity_and_ones():
    M = K = 48
    N = 40
    a, b = G.matmul_inputs(M, N, K, "f32", "identity")
    c = oracle.evaluate(S.matmul(M, N, K), [a, b])[0]
    assert np.array_equal(c, b.astype(np.float64))            # A = I ⇒ C = B exactly
    a, b = G.matmul_inputs(M, N, 300, "bf16", "ones")
    c = oracle.evaluate(S.matmul(M, N, 300, "bf16"), [a, b])[0]
    assert np.all(c == 300.0)                                  # ones·ones = K exactly


@pytest.mark.parametrize("dt", ["f32", "bf16"])
def test_matmul_vs_numpy(dt):
    M, N, K = 33, 47, 129
    a, b = G.matmul_inputs(M, N, K, dt)
    c = oracle.evaluate(S.matmul(M, N, K, dt), [a, b])[0]
    ref = f64(a, dt) @ f64(b, dt)
    assert np.max(np.abs(c - ref)) <= 1e-12 * np.max(np.abs(f64(a, dt)) @ np.abs(f64(b, dt)))


def test_matmul_transposed_and_batched():
    M, N, K = 10, 12, 9
    g = G.rng(1)
    a = g.uniform(-1, 1, (M, K)).astype(np.float32)
    bt = g.uniform(-1, 1, (N, K)).astype(np.float32)
    c = oracle.evaluate(S.matmul_t(M, N, K), [a, bt])[0]
    assert np.allclose(c, a.astype(np.float64) @ bt.astype(np.float64).T, rtol=0, atol=1e-13)
    B = 3
    a = g.uniform(-1, 1, (B, M, K)).astype(np.float32)
    b = g.uniform(-1, 1, (B, K, N)).astype(np.float32)
    c = oracle.evaluate(S.bmatmul(B, M, N, K), [a, b])[0]
    assert np.allclose(c, np.einsum("bik,bkj->bij", a.astype(np.float64), b.astype(np.float64)), atol=1e-13)


def test_matvec_vs_numpy():
    I, K = 17, 1000
    g = G.rng(3)
    m = g.uniform(-1, 1, (I, K)).astype(np.float32)
    v = g.uniform(-1, 1, (K,)).astype(np.float32)
    w = oracle.evaluate(S.matvec(I, K), [m, v])[0]
    assert np.allclose(w, m.astype(np.float64) @ v.astype(np.float64), rtol=0, atol=1e-12)


# ------------------------------------------------------------- Jacobi (C3)
def test_jacobi3d_golden_and_closed_forms():
    g = gold("jacobi3d.json")
    w = g["weights"]
    assert abs(sum(w.values()) - g["sum_w"]) < 1e-15
    Z, Y, X = 6, 7, 9
    sp = S.jacobi3d(Z, Y, X)
    v = oracle.evaluate(sp, G.jacobi3d_inputs(Z, Y, X, "constant"))[0]
    assert v.shape == (Z - 2, Y - 2, X - 2)
    assert np.allclose(v, g["constant_field_2_0"], rtol=0, atol=1e-14)
    u = G.jacobi3d_inputs(Z, Y, X, "linear")[0]
    v = oracle.evaluate(sp, [u])[0]
    uc = u[1:-1, 1:-1, 1:-1].astype(np.float64)
    closed = uc * g["sum_w"] + (w["xp"] - w["xm"]) + 2 * (w["yp"] - w["ym"]) + 3 * (w["zp"] - w["zm"])
    assert abs(((w["xp"] - w["xm"]) + 2 * (w["yp"] - w["ym"]) + 3 * (w["zp"] - w["zm"])) - g["linear_field_offset"]) < 1e-12
    assert np.allclose(v, closed, rtol=0, atol=1e-12)


def test_jacobi3d_vs_numpy_slicing():
    Z, Y, X = 7, 9, 11
    u = G.jacobi3d_inputs(Z, Y, X)[0]
    v = oracle.evaluate(S.jacobi3d(Z, Y, X), [u])[0]
    w = S.J3D_WEIGHTS
    U = u.astype(np.float64)
    c = U[1:-1, 1:-1, 1:-1]
    ref = (w["c"] * c + w["xm"] * U[1:-1, 1:-1, :-2] + w["xp"] * U[1:-1, 1:-1, 2:]
           + w["ym"] * U[1:-1, :-2, 1:-1] + w["yp"] * U[1:-1, 2:, 1:-1]
           + w["zm"] * U[:-2, 1:-1, 1:-1] + w["zp"] * U[2:, 1:-1, 1:-1])
    assert np.allclose(v, ref, rtol=0, atol=1e-13)


def test_gaussian2d_closed_forms_and_scipy():
    """Gaussian_2D (reading C-31): dyadic weights k/256 make the closed forms exact in fp64 —
    a constant field is reproduced, the symmetric window maps a linear field x + 2y to its
    value at the window centre; random images agree with scipy's 'valid' correlation."""
    import scipy.signal
    I, J = 9, 13
    sp = S.gaussian2d(I, J)
    assert abs(sum(sp["fparams"]) - 1.0) == 0.0
    v = oracle.evaluate(sp, G.gaussian2d_inputs(I, J, "constant"))[0]
    assert v.shape == (I, J) and np.all(v == 3.0)
    v = oracle.evaluate(sp, G.gaussian2d_inputs(I, J, "linear"))[0]
    jj, ii = np.meshgrid(np.arange(J), np.arange(I))
    assert np.array_equal(v, (jj + 2) + 2.0 * (ii + 2))
    img = G.gaussian2d_inputs(I, J)[0]
    w = np.outer(S.GAUSS5, S.GAUSS5) / 256.0
    ref = scipy.signal.correlate2d(img.astype(np.float64), w, mode="valid")
    v = oracle.evaluate(sp, [img])[0]
    assert np.allclose(v, ref, rtol=0, atol=1e-14)


def test_jacobi1d_three_accesses():
    K = 1000
    vin = G.rng(9).uniform(0, 1, K + 2).astype(np.float32)
    w = oracle.evaluate(S.jacobi1d(K), [vin])[0]
    a, b, c = S.J1D_WEIGHTS
    V = vin.astype(np.float64)
    assert np.allclose(w, a * V[:-2] + b * V[1:-1] + c * V[2:], rtol=0, atol=1e-14)


def test_cc_identity_is_copy():
    x = G.rng(4).uniform(-1, 1, (3, 4, 5)).astype(np.float32)
    y = oracle.evaluate(S.copy_spec([3, 4, 5]), [x])[0]
    assert np.array_equal(y, x.astype(np.float64))


# ----------------------------------------------------------- CCSD(T) (C4a)
def test_ccsd_sd1_vs_einsum():
    sp = S.ccsd_sd1(2, 3, "f32")
    t2, v2 = G.gen_inputs(sp, 4000)
    t3 = oracle.evaluate(sp, [t2, v2])[0]
    ref = np.einsum("gdab,gcfe->cbafed", t2.astype(np.float64), v2.astype(np.float64))
    assert np.allclose(t3, ref, rtol=0, atol=1e-14)


def test_ccsd_sd2_vs_einsum():
    sp = S.ccsd_sd2(h7=5, p4=3, p5=4, h1=3, h3=2, h2=3, p6=4)
    t2, v2 = G.gen_inputs(sp, 4000)
    t3 = oracle.evaluate(sp, [t2, v2])[0]
    # t3[h3,h2,h1,p6,p5,p4] = Σ_h7 t2[h7,p4,p5,h1] v2[h3,h2,p6,h7]
    ref = np.einsum("gdea,cbfg->cbafed", t2.astype(np.float64), v2.astype(np.float64))
    assert np.allclose(t3, ref, rtol=0, atol=1e-14)


# --------------------------------------------------------------- MCC (C4b)
def test_mcc_vs_torch_conv2d():
    torch = pytest.importorskip("torch")
    N, P, Q, K, R, Sx, C = 2, 3, 4, 5, 3, 3, 2
    sp = S.mcc(N, P, Q, K, R, Sx, C, "f32")
    img, flt = G.mcc_inputs(sp)
    res = oracle.evaluate(sp, [img, flt])[0]
    x = torch.from_numpy(img.astype(np.float64)).permute(0, 3, 1, 2)      # NHWC → NCHW
    w = torch.from_numpy(flt.astype(np.float64)).permute(0, 3, 1, 2)      # KRSC → KCRS
    ref = torch.nn.functional.conv2d(x, w, stride=2)[:, :, :P, :Q].permute(0, 2, 3, 1).numpy()
    assert res.shape == ref.shape
    assert np.allclose(res, ref, rtol=0, atol=1e-13)


def test_mcc_caps_vs_strided_einsum():
    """MCC_Caps (reading C-33): numpy strided-window view of the image + einsum over
    (r, s, c, l) with the 4×4 capsule matrix product; with 1×1 capsules it is MCC and
    matches torch conv2d."""
    N, P, Q, K, R, Sx, C = 2, 3, 2, 3, 3, 3, 2
    sp = S.mcc_caps(N, P, Q, K, R, Sx, C, 2, 3, 4)
    img, flt = G.gen_inputs(sp, 4200)
    res = oracle.evaluate(sp, [img, flt])[0]
    X = img.astype(np.float64)
    win = np.lib.stride_tricks.sliding_window_view(X, (R, Sx), axis=(1, 2))[:, ::2, ::2]
    win = win[:, :P, :Q]                                   # [n,p,q,c,i,l,r,s]
    ref = np.einsum("npqcilrs,krsclj->npqkij", win, flt.astype(np.float64))
    assert res.shape == ref.shape
    assert np.allclose(res, ref, rtol=0, atol=1e-13)
    torch = pytest.importorskip("torch")
    sp1 = S.mcc_caps(N, P, Q, K, R, Sx, C, 1, 1, 1)
    img1, flt1 = G.gen_inputs(sp1, 4210)
    r1 = oracle.evaluate(sp1, [img1, flt1])[0][..., 0, 0]
    x = torch.from_numpy(img1[..., 0, 0].astype(np.float64)).permute(0, 3, 1, 2)
    w = torch.from_numpy(flt1[..., 0, 0].astype(np.float64)).permute(0, 3, 1, 2)
    ref1 = torch.nn.functional.conv2d(x, w, stride=2)[:, :, :P, :Q].permute(0, 2, 3, 1).numpy()
    assert np.allclose(r1, ref1, rtol=0, atol=1e-13)


# --------------------------------------------------------------- PRL (C5)
def _prl_numpy(new, db, dbid, wa, wd, op):
    """Independent vectorised formulation (SURVEY §8(c).4 PRL row): broadcast compare,
    weights via a 256-entry table, argmax via np.lexsort / the literal rule."""
    N, I = new[0].shape[0], db[0].shape[0]
    mask = np.zeros((N, I), np.int64)
    for k in range(8):
        mask |= (new[k][:, None] == db[k][None, :]).astype(np.int64) << k
    table = np.zeros(256)
    for m in range(256):
        acc = 0.0
        for k in range(8):
            acc = acc + (wa[k] if (m >> k) & 1 else wd[k])
        table[m] = acc
    wt = table[mask]
    pc = np.zeros_like(mask)
    for k in range(8):
        pc += (mask >> k) & 1
    idm = np.where(mask == 255, 14, pc)
    out = []
    for n in range(N):
        if op == "PW_PRL_ARGMAX":
            order = np.lexsort((dbid, wt[n], (idm[n] == 14).astype(np.int64)))
            i = order[-1]
        else:   # literal rule ⇒ last record with id 14, else the last record
            hits = np.nonzero(idm[n] == 14)[0]
            i = hits[-1] if len(hits) else I - 1
        out.append((dbid[i], wt[n, i], idm[n, i]))
    return out


@pytest.mark.parametrize("op", ["PW_PRL_ARGMAX", "PW_PRL_PAPER"])
def test_prl_tiny_golden(op):
    g = gold("prl_tiny.json")
    ins, (wa, wd) = G.prl_tiny()
    assert wa == g["wa"] and wd == g["wd"]
    mid, mw, idm = oracle.evaluate(S.prl(3, 4, op, weights=(wa, wd)), ins)
    for n, (e_id, e_w, e_m) in enumerate(g[op]):
        assert (mid[n], mw[n], idm[n]) == (e_id, e_w, e_m)


@pytest.mark.parametrize("op", ["PW_PRL_ARGMAX", "PW_PRL_PAPER"])
def test_prl_bruteforce_64(op):
    N = I = 64
    ins = G.prl_inputs(N, I, seed_base=5100, dup_frac=0.7)
    # small domains so that many partial and exact matches occur
    ins = [(x % 3).astype(np.uint32) if k < 16 else x for k, x in enumerate(ins)]
    wa, wd = S.prl_weights()
    mid, mw, idm = oracle.evaluate(S.prl(N, I, op), ins)
    ref = _prl_numpy(ins[:8], ins[8:16], ins[16], wa, wd, op)
    for n in range(N):
        assert (mid[n], mw[n], idm[n]) == ref[n]


def test_prl_planted_duplicates():
    N, I = 256, 512
    ins = G.prl_inputs(N, I, seed_base=5200, dup_frac=1.0, redraw_p=0.0)
    wa, wd = S.prl_weights()
    mid, mw, idm = oracle.evaluate(S.prl(N, I), ins)
    assert np.all(idm == 14)
    acc = 0.0
    for w in wa:                     # fp64 left fold in field order (reading C-18);
        acc = acc + w                # NB: Python 3.12 sum() is compensated, not a fold
    assert np.all(mw == acc)
    table = {}
    for k in range(256):
        acc = 0.0
        for f in range(8):
            acc = acc + (wa[f] if (k >> f) & 1 else wd[f])
        table[acc] = k
    ins2 = G.prl_inputs(N, I, seed_base=5300)
    _, mw2, _ = oracle.evaluate(S.prl(N, I), ins2)
    assert all(w in table for w in mw2.tolist())     # weight ∈ {Σ_k sel_k} over 256 masks


# ------------------------------------------------- overwrite / coverage / errors
def test_outputs_outside_image_untouched():
    d = ["i"]
    sp = S.make_spec("strided", d, [5], ["CC"], "IDENTITY",
                     [S.buffer("x", "f32", [["i"]], d)],
                     [S.buffer("y", "f32", [["2*i"]], d, shape=[10])])
    x = np.arange(5, dtype=np.float32)
    y = oracle.evaluate(sp, [x], fill=-7.0)[0]
    assert np.array_equal(y[0::2], x.astype(np.float64))
    assert np.all(y[1::2] == -7.0)


def test_invalid_specs_rejected():
    d = ["i"]
    bad_neg = S.make_spec("neg", d, [4], ["CC"], "IDENTITY", [S.buffer("x", "f32", [["i-1"]], d)],
                          [S.buffer("y", "f32", [["i"]], d)])
    with pytest.raises(oracle.OracleError):
        oracle.evaluate(bad_neg, [np.zeros(4, np.float32)])
    small = S.make_spec("small", d, [4], ["CC"], "IDENTITY", [S.buffer("x", "f32", [["i"]], d, shape=[3])],
                        [S.buffer("y", "f32", [["i"]], d)])
    with pytest.raises(oracle.OracleError):
        oracle.shapes(small)
    noninj = S.make_spec("noninj", ["i", "j"], [3, 3], ["CC", "CC"], "IDENTITY",
                         [S.buffer("x", "f32", [["i", "j"]], ["i", "j"])],
                         [S.buffer("y", "f32", [["i+j"]], ["i", "j"])])
    with pytest.raises(oracle.OracleError):
        oracle.evaluate(noninj, [np.zeros((3, 3), np.float32)])


def test_bf16_rounding_matches_torch():
    torch = pytest.importorskip("torch")
    x = G.rng(11).uniform(-3, 3, 100000).astype(np.float32)
    bits = G.f32_to_bf16_bits(x)
    tb = torch.from_numpy(x).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(bits, tb)


def test_sampled_points_equal_full():
    sp = S.matmul(20, 30, 17)
    a, b = G.matmul_inputs(20, 30, 17)
    full = oracle.evaluate(sp, [a, b])[0]
    pts = oracle.random_points(sp, 50)
    lin, vals = oracle.evaluate_points(sp, [a, b], pts)
    assert np.array_equal(full.ravel()[lin[0]], vals[0])
    sp = S.prl(16, 40)
    ins = G.prl_inputs(16, 40)
    full = oracle.evaluate(sp, ins)
    lin, vals = oracle.evaluate_points(sp, ins, oracle.random_points(sp, 10))
    for b in range(3):
        assert np.array_equal(full[b].ravel()[lin[b]], vals[b])


# ------------------------------------------------------------------ F3: stencil time-stepping
def _j3d_numpy_sweeps(u0, sweeps):
    """Independent formulation (numpy slicing, fp64) of reading C-34: interior update by the
    seven shifted slabs of SURVEY §8(d) D-3 / reading C-16, boundary shell kept."""
    w = S.J3D_WEIGHTS
    u = u0.astype(np.float64).copy()
    for _ in range(sweeps):
        v = u.copy()
        v[1:-1, 1:-1, 1:-1] = (w["c"] * u[1:-1, 1:-1, 1:-1]
                               + w["xm"] * u[1:-1, 1:-1, :-2] + w["xp"] * u[1:-1, 1:-1, 2:]
                               + w["ym"] * u[1:-1, :-2, 1:-1] + w["yp"] * u[1:-1, 2:, 1:-1]
                               + w["zm"] * u[:-2, 1:-1, 1:-1] + w["zp"] * u[2:, 1:-1, 1:-1])
        u = v
    return u


def test_stencil_sweeps_pins():
    """oracle.stencil_sweeps (reading C-34) against: the single-sweep Jacobi_3D oracle (T=1,
    interior), the numpy slicing formulation (T=3), the closed form c·(Σw)^T at points farther
    than T from the boundary of a constant field, and the domain of dependence (a perturbation
    at p changes nothing farther than T away after T sweeps)."""
    Z, Y, X = 9, 10, 11
    u0 = np.random.Generator(np.random.PCG64(3401)).random((Z, Y, X)).astype(np.float32)
    sp = S.jacobi3d_sweep(Z, Y, X)
    one = oracle.stencil_sweeps(sp, u0, 1)
    ref1 = oracle.evaluate(S.jacobi3d(Z, Y, X), [u0])[0].reshape(Z - 2, Y - 2, X - 2)
    assert np.array_equal(one[1:-1, 1:-1, 1:-1], ref1)
    assert np.array_equal(one[0], u0[0].astype(np.float64)) and np.array_equal(one[:, :, -1], u0[:, :, -1].astype(np.float64))
    three = oracle.stencil_sweeps(sp, u0, 3)
    np.testing.assert_allclose(three, _j3d_numpy_sweeps(u0, 3), rtol=0, atol=1e-12)
    # constant field: centre after T sweeps is c·(Σw)^T (distance to the shell > T)
    c = 2.0
    T = 3
    const = oracle.stencil_sweeps(sp, np.full((Z, Y, X), c, np.float32), T)
    sw = sum(S.J3D_WEIGHTS.values())
    assert abs(const[4, 4, 5] - c * sw ** T) <= 1e-12
    # domain of dependence (Manhattan distance ≤ T for the 7-point cross)
    u1 = u0.copy()
    u1[4, 5, 5] += 1.0
    d = np.abs(oracle.stencil_sweeps(sp, u1, 2) - oracle.stencil_sweeps(sp, u0, 2))
    zz, yy, xx = np.nonzero(d)
    assert len(zz) and (np.abs(zz - 4) + np.abs(yy - 5) + np.abs(xx - 5)).max() <= 2


def test_z_slabs_partition():
    for Z, world in ((10, 1), (10, 3), (512, 8), (9, 7)):
        sl = S.z_slabs(Z, world)
        assert sl[0][0] == 1 and sl[-1][1] == Z - 1
        assert all(a[1] == b[0] for a, b in zip(sl, sl[1:]))
        sizes = [hi - lo for lo, hi in sl]
        assert max(sizes) - min(sizes) <= 1 and min(sizes) >= 1
