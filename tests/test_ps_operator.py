"""The prefix-sum combine operator ps(add) (Listing 17) and MBBS (reading
C-30): oracle pins (CPU) and GPU parity (T6 scan, T0 generic)."""
import copy

import numpy as np
import pytest

import oracle
from mdh_workloads import gen as G
from mdh_workloads import specs as S


# --------------------------------------------------------------------- oracle pins
@pytest.mark.parametrize("shape,dim", [([1000], 0), ([5, 1000], 1), ([300, 7], 0), ([3, 4, 5], 1)])
def test_prefix_sum_vs_numpy_cumsum(shape, dim):
    x = G.rng(3).uniform(-1, 1, shape).astype(np.float32)
    y = oracle.evaluate(S.prefix_sum(shape, dim), [x])[0]
    # both are sequential left folds in fp64, so they agree exactly
    assert np.array_equal(y, np.cumsum(x.astype(np.float64), axis=dim))


def test_prefix_sum_int32_wraps():
    x = G.rng(4).integers(-2 ** 31, 2 ** 31, 5000, dtype=np.int64).astype(np.int32)
    y = oracle.evaluate(S.prefix_sum([5000], 0, "i32"), [x])[0]
    ref = (np.cumsum(x.astype(np.int64)) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    assert np.array_equal(y, ref)


def test_mbbs_closed_form():
    X = G.rng(5).integers(-100, 100, (64, 37)).astype(np.int32)
    r = oracle.evaluate(S.mbbs(64, 37, "i32"), [X])[0]
    assert np.array_equal(r, np.cumsum(X.astype(np.int64).sum(axis=0)))      # R[j] = Σ_{j'≤j} Σ_i X[i,j']
    ones = np.ones((10, 20), np.float32)
    r = oracle.evaluate(S.mbbs(10, 20), [ones])[0]
    assert np.array_equal(r, 10.0 * np.arange(1, 21))


def test_mbbs_both_orientations():
    """MBBS as (pw(add), ps(add)) over loops (i, j) and as (ps(add), pw(add)) over loops
    (j, i) (SURVEY §8(f) F1's orientation): the same closed form R[j] = Σ_{j'≤j} Σ_i X[i,j']
    — exactly for int32, and to fp64 rounding for floats (the fold orders differ)."""
    X = G.rng(7).integers(-1000, 1000, (33, 29)).astype(np.int32)
    ref = np.cumsum(X.astype(np.int64).sum(axis=0))
    for order in ("pw_ps", "ps_pw"):
        assert np.array_equal(oracle.evaluate(S.mbbs(33, 29, "i32", order), [X])[0], ref)
    Xf = G.rng(8).uniform(-1, 1, (33, 29)).astype(np.float32)
    a = oracle.evaluate(S.mbbs(33, 29, "f32", "pw_ps"), [Xf])[0]
    b = oracle.evaluate(S.mbbs(33, 29, "f32", "ps_pw"), [Xf])[0]
    exact = np.array([sum(float(v) for v in Xf[:, :j + 1].ravel()) for j in range(29)])
    assert np.max(np.abs(a - exact)) < 1e-12 and np.max(np.abs(b - exact)) < 1e-12


def test_ps_homomorphism_split():
    """Listing 17 for a contiguous split P|Q of the ps dim: res[P] = lhs, res[q] = lhs[max P] ⊕ rhs[q]."""
    n, s = 1000, 377
    x = G.rng(6).uniform(-1, 1, n).astype(np.float32)
    spec = S.prefix_sum([n], 0)
    full = oracle.evaluate(spec, [x])[0]
    lo = oracle.evaluate(S.prefix_sum([s], 0), [x[:s].copy()])[0]
    hi = oracle.evaluate(S.prefix_sum([n - s], 0), [x[s:].copy()])[0]
    comb = np.concatenate([lo, lo[-1] + hi])
    assert np.max(np.abs(comb - full)) <= 1e-12 * np.max(np.abs(np.cumsum(np.abs(x.astype(np.float64)))))


# --------------------------------------------------------------------- GPU parity
gpu = pytest.mark.gpu


@gpu
@pytest.mark.parametrize("shape,dim,dt", [([1], 0, "f32"), ([1000], 0, "f32"), ([(1 << 20) + 7], 0, "f32"),
                                          ([5, 4096], 1, "f32"), ([64, 9000], 1, "i32"), ([300, 7], 0, "f32"),
                                          ([3, 4, 5], 1, "i32")])
def test_gpu_prefix_sum(shape, dim, dt):
    # the literal oracle folds [0, k] for every k (O(n^2) per row): sample long rows
    from gpu_util import assert_close_full, assert_close_points, run_gpu
    spec = S.prefix_sum(shape, dim, dt)
    x = G.gen_inputs(spec, 6100, "positive")
    got, p = run_gpu(spec, x)
    assert p.template == "T6_prefix_scan"
    tol, kind = (1e-4, "rel") if dt == "f32" else (0, "exact")
    if shape[dim] <= 10000:
        assert_close_full(spec, x, got, tol, kind=kind)
    else:
        assert_close_points(spec, x, got, tol, n=64, kind=kind)
        assert abs(float(got[0][-1]) - float(np.sum(x[0].astype(np.float64)))) <= 1e-4 * float(np.sum(x[0]))


@gpu
@pytest.mark.parametrize("shape,dt,tile", [([3, 200000], "i32", None), ([3, 100003], "f32", None),
                                           ([2, 300001], "f64", "seg=4096"), ([1 << 22], "i64", "seg=65536"),
                                           ([1 << 22], "u32", None), ([5, 65536 * 3 + 4096 * 5 + 1], "f32", None),
                                           ([(1 << 24) + 12345], "f32", None), ([3, 100003], "f32", "seg=8192"),
                                           ([(1 << 25) + 3], "f32", None), ([7, 3000017], "i32", None)])
def test_gpu_single_pass_scan(shape, dt, tile):
    """Long rows take a single-pass scan: the tree scan (default; per-row tree of tile
    aggregates) or the segmented one (tile knob seg): aligned and misaligned row starts,
    ragged tile counts, several rows, integer wrap-around exact, repeatable."""
    from gpu_util import run_gpu
    spec = S.prefix_sum(shape, len(shape) - 1, dt)
    x = G.gen_inputs(spec, 6150, "signed" if dt in ("f32", "f64") else "positive")
    got, p = run_gpu(spec, x, force_tile=tile)
    assert p.template == "T6_prefix_scan" and (p.describe()["tiles"]["seg"] > 0) == (tile is not None)
    x0 = x[0].reshape(shape)
    if dt in ("f32", "f64"):
        ref = np.cumsum(x0.astype(np.float64), axis=-1)
        scale = np.cumsum(np.abs(x0.astype(np.float64)), axis=-1)
        assert np.max(np.abs(got[0].reshape(shape) - ref) / scale) <= (1e-4 if dt == "f32" else 1e-12)
    else:   # two's-complement wrap: cumsum in the same width is exact
        ref = np.cumsum(x0, axis=-1, dtype=x0.dtype)
        assert np.array_equal(got[0].reshape(shape), ref)
    for _ in range(2):                         # repeatable (deterministic association, epochs)
        got2, _ = run_gpu(spec, x, plan=p)
        assert np.array_equal(got[0], got2[0])


@gpu
@pytest.mark.parametrize("IJ", [(64, 37), (1000, 5000), (4096, 8192), (8192, 8192), (300, 1000), (40, 64),
                                (64, 4096), (16, 32768), (8, 12288)])
def test_gpu_mbbs(IJ):
    """MBBS on T6; shapes with J % 4 == 0 take the column-fold K1 (16-byte column loads,
    the row range split over blocks, ordered ticket fold; ragged last column group for
    J = 1000); J = 4096·nv (nv = 1, 2, 3, 8) then take the register row scan launched as a
    programmatic dependent of the fold.  Run twice on one plan: tickets back at rest,
    results bit-identical."""
    from gpu_util import assert_close_full, run_gpu
    spec = S.mbbs(*IJ)
    x = G.gen_inputs(spec, 6200, "positive")
    got, p = run_gpu(spec, x)
    assert p.template == "T6_prefix_scan"
    if IJ[0] * IJ[1] <= 64 * 64:
        assert_close_full(spec, x, got, 1e-4, kind="rel")
    else:   # closed form R[j] = Σ_{j'≤j} Σ_i X[i,j'] (pinned against the oracle above)
        ref = np.cumsum(x[0].astype(np.float64).sum(axis=0))
        assert np.max(np.abs(got[0] - ref) / ref) <= 1e-4
    got2, _ = run_gpu(spec, x, plan=p)
    assert np.array_equal(got[0], got2[0])


@gpu
@pytest.mark.parametrize("IJ", [(64, 37), (1000, 5000), (8192, 8192)])
def test_gpu_mbbs_ps_pw_orientation(IJ):
    """MBBS with the loops swapped — md_hom[J,I](id, (ps(add), pw(add))) — against the
    oracle (small) or the closed form (large)."""
    from gpu_util import assert_close_full, run_gpu
    spec = S.mbbs(*IJ, order="ps_pw")
    x = G.gen_inputs(spec, 6250, "positive")
    got, p = run_gpu(spec, x)
    assert p.template == "T6_prefix_scan"
    if IJ[0] * IJ[1] <= 64 * 64:
        assert_close_full(spec, x, got, 1e-4, kind="rel")
    else:
        ref = np.cumsum(x[0].astype(np.float64).sum(axis=0))
        assert np.max(np.abs(got[0] - ref) / ref) <= 1e-4


@gpu
def test_gpu_two_ps_dims_generic():
    """Two ps dims (a 2-D summed-area table) fall back to the generic template (T0)."""
    from gpu_util import assert_close_full, run_gpu
    d = ["i", "j"]
    spec = S.make_spec("sat", d, [40, 50], ["PS_ADD", "PS_ADD"], "IDENTITY",
                       [S.buffer("x", "f32", [["i", "j"]], d)], [S.buffer("y", "f32", [["i", "j"]], d)])
    x = G.gen_inputs(spec, 6300, "positive")
    got, p = run_gpu(spec, x)
    assert p.template == "T0_generic"
    ref = np.cumsum(np.cumsum(x[0].astype(np.float64), 0), 1)
    assert np.max(np.abs(got[0] - ref) / ref) <= 1e-4
    assert_close_full(spec, x, got, 1e-4, kind="rel")
