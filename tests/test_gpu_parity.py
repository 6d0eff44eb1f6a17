"""GPU parity: the CUDA path through the C-ABI vs the CPU oracle on the same seeded
inputs (SURVEY §8(c).5 parity matrix).  Tolerances (north star):
integers / indices / PRL / max-min selections bit-exact; fp32 1e-4 (element-wise on
positive data, scale-normalised on signed data, reading C-14); bf16 inputs 1e-2."""
import json
import os

import numpy as np
import pytest

import oracle
from mdh_workloads import gen as G
from mdh_workloads import specs as S

from gpu_util import assert_close_full, assert_close_points, run_gpu

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")


# ----------------------------------------------------------------- T2: Dot / MatVec
DOT_N = [1, 2, 3, 31, 32, 33, 127, 4097, 65537, 1 << 20, (1 << 20) + 3]


@pytest.mark.parametrize("N", DOT_N)
@pytest.mark.parametrize("op", ["PW_ADD", "PW_MAX", "PW_MIN"])
@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_dot(N, op, dt):
    spec = S.dot(N, dt, op)
    kind = "positive" if dt == "f32" and op == "PW_ADD" else "signed"
    x = G.dot_inputs(N, dt, kind)
    got, p = run_gpu(spec, x)
    assert p.template == "T2_reduce"
    if dt == "i32" or op != "PW_ADD":
        if dt == "f32":   # selections of fp32 products: only f's own fp32 rounding (≤2^-24)
            assert_close_full(spec, x, got, 1e-6, kind="rel")
        else:
            assert_close_full(spec, x, got, 0, kind="exact")
    else:
        assert_close_full(spec, x, got, 1e-4, kind="rel")


def test_dot_signed_fp32_scale_normalised():
    N = 1 << 20
    x = G.dot_inputs(N, "f32", "signed")
    got, _ = run_gpu(S.dot(N, "f32"), x)
    assert_close_full(S.dot(N, "f32"), x, got, 1e-4, kind="scale")


def test_dot_int32_golden():
    with open(os.path.join(GOLD, "dot_int32.json")) as f:
        g = json.load(f)
    N = g["N"]
    for kind in ("iota_one", "iota_iota"):
        got, _ = run_gpu(S.dot(N, "i32"), G.dot_inputs(N, "i32", kind))
        assert int(got[0][0]) == g[kind]


def test_dot_repeatable_bit_identical():
    N = (1 << 20) + 3
    x = G.dot_inputs(N, "f32", "signed")
    a, p = run_gpu(S.dot(N, "f32"), x)
    b, _ = run_gpu(S.dot(N, "f32"), x, plan=p)
    assert a[0].tobytes() == b[0].tobytes()


@pytest.mark.parametrize("I,K", [(1, 1), (3, 1000), (17, 1 << 20), (4096, 4096), (8192, 8192)])
def test_matvec(I, K):
    spec = S.matvec(I, K)
    x = G.gen_inputs(spec, 2100, "positive")
    got, p = run_gpu(spec, x)
    assert p.template == "T2_reduce"
    assert_close_full(spec, x, got, 1e-4, kind="rel")


@pytest.mark.parametrize("I,K", [(1, 1024), (37, 2048), (1000, 4096), (4096, 4096), (8192, 8192), (300, 8192)])
@pytest.mark.parametrize("tile", ["mode=3", "mode=3,per_thread=4"])
def test_matvec_row_range(I, K, tile):
    """Row-range MatVec kernel (tile knob mode 3: contiguous row ranges per CTA, x held in
    registers): ragged row ranges (I not a multiple of the grid or of 8), every supported
    row length, fp32 1e-4 vs the fp64 oracle."""
    spec = S.matvec(I, K)
    x = G.gen_inputs(spec, 2150, "positive")
    got, p = run_gpu(spec, x, force_tile=tile)
    assert "row-range" in p.describe()["why"], p.describe()["why"]
    assert_close_full(spec, x, got, 1e-4, kind="rel")


@pytest.mark.parametrize("op", ["PW_MAX", "PW_MIN"])
def test_matvec_row_range_maxmin(op):
    spec = S.matvec(777, 2048, "f32", op)
    x = G.gen_inputs(spec, 2160, "signed")
    got, p = run_gpu(spec, x, force_tile="mode=3")
    assert "row-range" in p.describe()["why"]
    assert_close_full(spec, x, got, 1e-6, kind="rel")


@pytest.mark.parametrize("op", ["PW_MAX", "PW_MIN", "PW_ADD"])
def test_matvec_int32(op):
    spec = S.matvec(37, 5001, "i32", op)
    x = G.gen_inputs(spec, 2200)
    got, _ = run_gpu(spec, x)
    assert_close_full(spec, x, got, 0, kind="exact")


@pytest.mark.parametrize("shape,red", [([1000, 37], [0]), ([5, 6, 7], [1]), ([64, 3], [0]), ([3, 100000], [1])])
def test_reductions_identity_f(shape, red):
    spec = S.reduce_spec(shape, red, "PW_ADD")
    x = G.gen_inputs(spec, 2300, "positive")
    got, _ = run_gpu(spec, x)
    assert_close_full(spec, x, got, 1e-4, kind="rel")


# ----------------------------------------------------------------- T1: stencils
@pytest.mark.parametrize("zyx", [(3, 3, 3), (5, 7, 9), (66, 130, 258)])
def test_jacobi3d(zyx):
    spec = S.jacobi3d(*zyx)
    x = G.jacobi3d_inputs(*zyx)
    got, p = run_gpu(spec, x)
    assert p.template == "T1_stencil"
    assert_close_full(spec, x, got, 1e-4, kind="scale")


def test_jacobi3d_full_size_sampled_and_closed_forms():
    spec = S.jacobi3d(512, 512, 512)
    x = G.jacobi3d_inputs(512, 512, 512)
    got, _ = run_gpu(spec, x)
    assert_close_points(spec, x, got, 1e-4, n=20000, kind="scale")
    with open(os.path.join(GOLD, "jacobi3d.json")) as f:
        g = json.load(f)
    got, _ = run_gpu(spec, G.jacobi3d_inputs(512, 512, 512, "constant"))
    assert np.abs(got[0].astype(np.float64) - g["constant_field_2_0"]).max() <= 1e-4 * 2.0 * 2.0 * 1.67


@pytest.mark.parametrize("zyx", [(5, 7, 9), (66, 130, 258)])
def test_jacobi3d_l2_prefetch_hint_variants(zyx):
    """Tile knob l2pf (L2 prefetch-size hint on the 7-point row loads): a cache hint only, so
    every setting is bit-identical to the others and within 1e-4 of the oracle."""
    spec = S.jacobi3d(*zyx)
    x = G.jacobi3d_inputs(*zyx)
    outs = []
    for pf in (0, 1, 2):
        got, p = run_gpu(spec, x, force_tile=f"zchunk=8,l2pf={pf}")
        assert p.template == "T1_stencil"
        outs.append(got[0])
    assert outs[0].tobytes() == outs[1].tobytes() == outs[2].tobytes()
    assert_close_full(spec, x, [outs[2]], 1e-4, kind="scale")


@pytest.mark.parametrize("IJ", [(1, 1), (3, 5), (17, 33), (224, 224), (129, 1030)])
def test_gaussian2d(IJ):
    """Gaussian_2D 5×5 (reading C-31; Fig 3) on the 2-D box-window T1 kernel:
    ragged x (non-multiple of 4, unaligned rows) and y-chunk tails."""
    I, J = IJ
    spec = S.gaussian2d(I, J)
    x = G.gaussian2d_inputs(I, J)
    got, p = run_gpu(spec, x)
    assert p.template == "T1_stencil"
    assert "box-window" in p.describe()["why"] or I * J < 4
    assert_close_full(spec, x, got, 1e-4, kind="rel")


def test_gaussian2d_full_size_closed_forms():
    I = J = 4096
    spec = S.gaussian2d(I, J)
    got, _ = run_gpu(spec, G.gaussian2d_inputs(I, J, "constant"))
    assert np.allclose(got[0], 3.0, rtol=1e-6, atol=0)
    x = G.gaussian2d_inputs(I, J)
    got, _ = run_gpu(spec, x)
    assert_close_points(spec, x, got, 1e-4, n=20000, kind="rel")


@pytest.mark.parametrize("K", [1, 3, 1000])
def test_jacobi1d(K):
    spec = S.jacobi1d(K)
    x = [G.rng(17).uniform(0, 1, K + 2).astype(np.float32)]
    got, _ = run_gpu(spec, x)
    assert_close_full(spec, x, got, 1e-4, kind="rel")


def test_copy_identity():
    spec = S.copy_spec([7, 33, 65])
    x = G.gen_inputs(spec, 2400)
    got, _ = run_gpu(spec, x)
    assert np.array_equal(got[0], x[0])


@pytest.mark.parametrize("dt", ["u32", "i64"])
@pytest.mark.parametrize("op", ["PW_ADD", "PW_MAX", "PW_MIN"])
def test_dot_u32_i64_wrap_and_order(dt, op):
    """uint32 (mod 2^32, unsigned order) and int64 (mod 2^64) reductions on T2, bit-exact
    against the oracle's u32 / i64 kinds (pinned against Python integers on the CPU)."""
    g = np.random.Generator(np.random.PCG64(62))
    n = 100003
    if dt == "u32":
        a = g.integers(0, 2 ** 32, n, dtype=np.uint64).astype(np.uint32)
        b = g.integers(0, 2 ** 32, n, dtype=np.uint64).astype(np.uint32)
    else:
        a = g.integers(-2 ** 40, 2 ** 40, n).astype(np.int64)
        b = g.integers(-2 ** 30, 2 ** 30, n).astype(np.int64)
    spec = S.dot(n, dt, op)
    got, _ = run_gpu(spec, [a, b])
    assert_close_full(spec, [a, b], got, 0, kind="exact")


# ----------------------------------------------------------------- T3: SIMT contraction
@pytest.mark.parametrize("mnk", [(1, 1, 1), (3, 5, 7), (127, 129, 65), (128, 256, 64), (300, 200, 1000)])
def test_matmul_fp32(mnk):
    M, N, K = mnk
    spec = S.matmul(M, N, K)
    x = G.matmul_inputs(M, N, K, "f32", "positive")
    got, p = run_gpu(spec, x)
    # degenerate 1-point dims carry no M/N group, so (1,1,1) is a plain reduction
    assert p.template == ("T2_reduce" if M == 1 or N == 1 else "T3_simt_contraction")
    assert_close_full(spec, x, got, 1e-4, kind="rel")


@pytest.mark.parametrize("mnk", [(3, 5, 7), (127, 129, 65), (128, 256, 64), (300, 200, 1000), (1000, 777, 333)])
def test_matmul_fp32_ffma2(mnk):
    """T3 SGEMM with the accumulators as fp32 pairs (FFMA2, the default; tile knob mode=0 the
    FFMA form): the same fp32 FMA sequence per element — bit-identical — and 1e-4 of the
    oracle."""
    M, N, K = mnk
    spec = S.matmul(M, N, K)
    x = G.matmul_inputs(M, N, K, "f32", "signed")
    for st in ("stages=4", "stages=2"):       # two CTAs per SM (default) / fragment-pipelined
        got, p = run_gpu(spec, x, force_tile=st + ",mode=1")
        ref, _ = run_gpu(spec, x, force_tile=st + ",mode=0")
        assert p.template == "T3_simt_contraction"
        assert np.array_equal(got[0], ref[0])
        assert_close_full(spec, x, got, 1e-4, kind="scale")


def test_matmul_fp32_full_size_sampled():
    spec = S.matmul(4096, 4096, 4096)
    x = G.matmul_inputs(4096, 4096, 4096, "f32", "signed")
    got, _ = run_gpu(spec, x)
    assert_close_points(spec, x, got, 1e-4, n=3000, kind="scale")
    x = G.matmul_inputs(4096, 4096, 4096, "f32", "ones")
    got, _ = run_gpu(spec, x)
    assert np.all(got[0] == 4096.0)


def test_matmul_identity_exact():
    spec = S.matmul(256, 384, 256)
    x = G.matmul_inputs(256, 384, 256, "f32", "identity")
    got, _ = run_gpu(spec, x)
    assert np.array_equal(got[0], x[1])


def test_matmul_int32_wraps():
    spec = S.matmul(70, 90, 300, "i32", "i32")
    x = G.gen_inputs(spec, 2500)
    got, _ = run_gpu(spec, x)
    assert_close_full(spec, x, got, 0, kind="exact")


def test_matmul_transposed_batched():
    spec = S.matmul_t(64, 500, 64)      # Fig 3 MatMul^T sizes
    x = G.gen_inputs(spec, 2600, "positive")
    got, _ = run_gpu(spec, x)
    assert_close_full(spec, x, got, 1e-4, kind="rel")
    spec = S.bmatmul(16, 10, 500, 64)   # Fig 3 bMatMul sizes
    x = G.gen_inputs(spec, 2700, "positive")
    got, _ = run_gpu(spec, x)
    assert_close_full(spec, x, got, 1e-4, kind="rel")


def test_ccsd_small_and_paper_inp1():
    spec = S.ccsd_sd1(2, 3, "f32")
    x = G.gen_inputs(spec, 4000)
    got, _ = run_gpu(spec, x)
    assert_close_full(spec, x, got, 1e-4, kind="scale")
    spec = S.ccsd_sd2()                 # paper Inp.1 reading (C-22), fp32
    x = G.gen_inputs(spec, 4001)
    got, _ = run_gpu(spec, x)
    assert_close_points(spec, x, got, 1e-4, n=5000, kind="scale")


def test_ccsd_full_size_fp32_sampled():
    spec = S.ccsd_sd1(24, 72, "f32")
    x = G.gen_inputs(spec, 4002)
    got, _ = run_gpu(spec, x)
    assert_close_points(spec, x, got, 1e-4, n=20000, kind="scale")


@pytest.mark.parametrize("cfg", [(2, 3, 4, 5, 3, 3, 2), (1, 7, 7, 512, 3, 3, 512), (1, 112, 112, 64, 7, 7, 3)])
def test_mcc_fp32(cfg):
    spec = S.mcc(*cfg, dtype="f32")
    x = G.mcc_inputs(spec)
    got, _ = run_gpu(spec, x)
    assert_close_full(spec, x, got, 1e-4, kind="scale")


@pytest.mark.parametrize("zyx", [(5, 7, 12), (66, 130, 260), (34, 19, 136), (64, 64, 64), (512, 512, 512)])
@pytest.mark.parametrize("tile", ["stages=3,zchunk=8", "stages=6,zchunk=16"])
def test_jacobi3d_tma_staged(zyx, tile):
    """The TMA-staged 7-point kernel (tile knob stages ≥ 3: input planes streamed into a
    shared-memory ring by cp.async.bulk.tensor; rows of a multiple of 4 floats, the
    kernel's eligibility): ragged x/y/z tiles, tiny grids, full
    size (sampled), against the oracle (scale-normalised 1e-4) and bit-identical to the
    register-queue kernel (same per-point arithmetic)."""
    Z, Y, X = zyx
    spec = S.jacobi3d(Z, Y, X)
    x = G.jacobi3d_inputs(Z, Y, X)
    got, p = run_gpu(spec, x, force_tile=tile)
    assert "tma" in p.describe()["why"], p.describe()["why"]
    ref, _ = run_gpu(spec, x, force_tile="stages=0")
    assert np.array_equal(got[0], ref[0])
    if Z * Y * X <= 66 * 130 * 258:
        assert_close_full(spec, x, got, 1e-4, kind="scale")
    else:
        assert_close_points(spec, x, got, 1e-4, n=20000, kind="scale")


# ----------------------------------------------------------------- T5: PRL
@pytest.mark.parametrize("op", ["PW_PRL_ARGMAX", "PW_PRL_PAPER"])
def test_prl_tiny_golden(op):
    with open(os.path.join(GOLD, "prl_tiny.json")) as f:
        g = json.load(f)
    ins, w = G.prl_tiny()
    spec = S.prl(3, 4, op, weights=w)
    got, p = run_gpu(spec, ins)
    assert p.template == "T5_prl_pairwise"
    for n, (e_id, e_w, e_m) in enumerate(g[op]):
        assert (int(got[0][n]), float(got[1][n]), int(got[2][n])) == (e_id, e_w, e_m)


@pytest.mark.parametrize("NI", [(1, 1), (64, 64), (1000, 777), (1 << 10, 1 << 15)])
@pytest.mark.parametrize("op", ["PW_PRL_ARGMAX", "PW_PRL_PAPER"])
def test_prl_full(NI, op):
    N, I = NI
    ins = G.prl_inputs(N, I, seed_base=5500)
    spec = S.prl(N, I, op)
    got, _ = run_gpu(spec, ins)
    assert_close_full(spec, ins, got, 0, kind="exact")


@pytest.mark.parametrize("R", [4, 8])
def test_prl_ties_full(R):
    """Rank ties (weights with equal sums for different masks, duplicated DB ids) through
    the id tie-break path, both register blockings (tile knob vec)."""
    N, I = 3000, 2500
    ins = G.prl_inputs(N, I, seed_base=5900)
    ins[16] = (ins[16] % 97).astype(np.int64)          # many equal ids
    wa, wd = [1.0, 1.0, 2.0, 2.0, 0.5, 0.5, 1.5, 1.5], [-1.0] * 8
    for op in ("PW_PRL_ARGMAX", "PW_PRL_PAPER"):
        spec = S.prl(N, I, op, weights=(wa, wd))
        got, p = run_gpu(spec, ins, force_tile=f"vec={R}")
        assert_close_full(spec, ins, got, 0, kind="exact")


# field codes around the fp16 edges of the packed compare (t5_prl.cu: code x is held as the
# fp16 pattern x < 0x7C00 ? x : x + 0x401): +0, subnormals, the first normal, the largest
# finite code, the codes remapped past the NaN range, and the last packable code
PRL_EDGE_CODES = np.array([0, 1, 2, 0x3FF, 0x400, 0x401, 0x7BFF, 0x7C00, 0x7C01, 0x7E00, 0x7FFF], np.uint32)


@pytest.mark.parametrize("case", ["edges_packed", "db_tile_unpackable", "new_unpackable", "all_unpackable"])
@pytest.mark.parametrize("op", ["PW_PRL_ARGMAX", "PW_PRL_PAPER"])
def test_prl_packed_and_general_paths(case, op):
    """Bit-exact on codes chosen to trip the packed fp16 compare (many agreements among
    the edge codes), and on inputs that force the per-field u32 compares: one DB tile with
    a code >= 2^15 (that tile alone, mid-fold), one new record with 0xFFFFFFFF (its whole
    CTA), and every code >= 2^15 (codes differing only above bit 15 must not agree)."""
    N, I = 1500, 1700
    ins = G.prl_inputs(N, I, seed_base=5700)
    g = np.random.Generator(np.random.PCG64(5799))
    for k in range(8):
        for b in (k, 8 + k):
            n = len(ins[b])
            pick = g.random(n) < 0.5
            ins[b] = np.where(pick, PRL_EDGE_CODES[g.integers(0, len(PRL_EDGE_CODES), n)], ins[b]).astype(np.uint32)
    if case == "db_tile_unpackable":
        ins[8 + 3][600] = 0x8000                      # DB tile 1 (records 512..1023)
    elif case == "new_unpackable":
        ins[5][1] = 0xFFFFFFFF
    elif case == "all_unpackable":
        for b in range(16):
            ins[b] = (ins[b] | np.uint32(0x10000) * (g.integers(0, 2, len(ins[b])).astype(np.uint32) + 1)).astype(np.uint32)
    spec = S.prl(N, I, op)
    got, p = run_gpu(spec, ins)
    assert p.template == "T5_prl_pairwise"
    assert_close_full(spec, ins, got, 0, kind="exact")


@pytest.mark.parametrize("NI", [(1 << 20, 1 << 14), (1 << 14, 1 << 20), (1 << 15, 1 << 15)])
def test_prl_config_sampled(NI):
    N, I = NI
    ins = G.prl_inputs(N, I, seed_base=5000)
    spec = S.prl(N, I)
    got, _ = run_gpu(spec, ins)
    assert_close_points(spec, ins, got, 0, n=400, kind="exact")


# ----------------------------------------------------------------- T0 and semantics
def test_generic_strided_output_untouched_elements():
    import torch
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device, to_numpy
    d = ["i", "k"]
    spec = S.make_spec("strided", d, [50, 30], ["CC", "PW_MAX"], "IDENTITY",
                       [S.buffer("x", "f32", [["i", "k"]], d)],
                       [S.buffer("y", "f32", [["3*i+1"]], d, shape=[151])])
    x = G.gen_inputs(spec, 2800)
    p = Plan(spec)
    y = torch.full((151,), -7.0, device="cuda")
    p([to_device(x[0], "f32", "cuda")], [y])
    torch.cuda.synchronize()
    yh = to_numpy(y, "f32")
    ref = oracle.evaluate(spec, x, fill=-7.0)[0]
    assert np.array_equal(yh.astype(np.float64), ref)


def test_generic_template_nonlinear_reduction():
    # pw dims not linear in the input (transposed) → T0 catch-all, still on the GPU
    d = ["a", "b", "c"]
    spec = S.make_spec("t0", d, [9, 5, 7], ["CC", "PW_ADD", "PW_ADD"], "IDENTITY",
                       [S.buffer("x", "f32", [["a", "c", "b"]], d)],
                       [S.buffer("y", "f32", [["a"]], d)])
    x = G.gen_inputs(spec, 2900, "positive")
    got, p = run_gpu(spec, x)
    assert p.template == "T0_generic"
    assert_close_full(spec, x, got, 1e-4, kind="rel")


def test_misaligned_pointer_rejected():
    import torch
    from paper_conf_sc_schulzegr25_b200 import Plan, MdhError
    p = Plan(S.dot(100, "f32"))
    a = torch.zeros(200, device="cuda")
    with pytest.raises(MdhError, match="INVALID_ARG"):
        p([a[1:101], a[100:]], [torch.zeros(4, device="cuda")])


# ----------------------------------------------------- homomorphism via virtual shards
def _virtual_shards(spec, inputs, world, shard_dim):
    """Run every rank's sub-domain plan on one GPU (MDH_PLAN_VIRTUAL_SHARD), slicing the
    inputs by the plan's local shapes; pw shards are recombined by mdh_combine_partials."""
    import torch
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device, to_numpy, VIRTUAL_SHARD
    parts, plans = [], []
    for r in range(world):
        p = Plan(spec, world_size=world, rank=r, shard_dim=shard_dim, flags=VIRTUAL_SHARD)
        tin = []
        for b, x in enumerate(inputs):
            shp, off, _ = p.local_shape(False, b)
            sl = tuple(slice(o, o + s) for o, s in zip(off, shp))
            tin.append(to_device(np.ascontiguousarray(x[sl]), spec["inputs"][b]["dtype"], "cuda"))
        outs = p.empty_outputs()
        p(tin, outs)
        parts.append((p, outs))
        plans.append(p)
    torch.cuda.synchronize()
    return parts


@pytest.mark.parametrize("world", [2, 3, 4, 8])
def test_virtual_shard_pw_dot_and_prl(world):
    from paper_conf_sc_schulzegr25_b200 import to_numpy
    N = 100003
    spec = S.dot(N, "i32")
    x = G.dot_inputs(N, "i32")
    parts = _virtual_shards(spec, x, world, 0)
    comb = parts[0][0].combine_partials([o for _, o in parts])
    assert int(to_numpy(comb[0], "i32")[0]) == int(oracle.evaluate(spec, x)[0][0])
    for op in ("PW_PRL_ARGMAX", "PW_PRL_PAPER"):
        spec = S.prl(300, 5000, op)
        ins = G.prl_inputs(300, 5000, seed_base=5600)
        parts = _virtual_shards(spec, ins, world, 1)
        comb = parts[0][0].combine_partials([o for _, o in parts])
        got = [to_numpy(c, b["dtype"]) for c, b in zip(comb, spec["outputs"])]
        assert_close_full(spec, ins, got, 0, kind="exact")


@pytest.mark.parametrize("world", [2, 3, 8])
def test_virtual_shard_cc_matmul_jacobi(world):
    from paper_conf_sc_schulzegr25_b200 import to_numpy
    spec = S.matmul(300, 200, 100)
    x = G.matmul_inputs(300, 200, 100, "f32", "positive")
    ref = oracle.evaluate(spec, x)[0]
    for p, outs in _virtual_shards(spec, x, world, 0):
        shp, off, _ = p.local_shape(True, 0)
        g = to_numpy(outs[0], "f32").astype(np.float64)
        r = ref[off[0]:off[0] + shp[0]]
        assert (np.abs(g - r) / np.abs(r)).max() <= 1e-4
    spec = S.jacobi3d(20, 12, 14)
    x = G.jacobi3d_inputs(20, 12, 14)
    ref = oracle.evaluate(spec, x)[0]
    for p, outs in _virtual_shards(spec, x, world, 0):
        shp, off, _ = p.local_shape(True, 0)
        g = to_numpy(outs[0], "f32").astype(np.float64)
        r = ref[off[0]:off[0] + shp[0]]
        assert np.abs(g - r).max() <= 1e-4 * 2


# ----------------------------------------------------------------- T4: tcgen05 contraction
def _mm_spec(M, N, K, a_t=False, b_t=False, out="f32"):
    d = ["i", "j", "k"]
    a = ["k", "i"] if a_t else ["i", "k"]
    b = ["j", "k"] if b_t else ["k", "j"]
    return S.make_spec("mm", d, [M, N, K], ["CC", "CC", "PW_ADD"], "MUL",
                       [S.buffer("A", "bf16", [a], d), S.buffer("B", "bf16", [b], d)],
                       [S.buffer("C", out, [["i", "j"]], d)])


@pytest.mark.parametrize("mnk", [(128, 256, 64), (256, 512, 128), (300, 200, 1000), (8, 8, 8), (1000, 1032, 72)])
@pytest.mark.parametrize("at,bt", [(False, False), (False, True), (True, False), (True, True)])
def test_matmul_bf16_tcgen05(mnk, at, bt):
    M, N, K = mnk
    spec = _mm_spec(M, N, K, at, bt)
    x = G.gen_inputs(spec, 3100, "positive")
    got, p = run_gpu(spec, x)
    # operands without a 16-byte aligned leading dimension are gathered into a TMA layout
    d = p.describe()
    lda = M if at else K
    ldb = K if bt else N
    assert p.template == "T4_tcgen05_contraction", d
    assert (d["t4_variant"] & 2 != 0) == (lda % 8 != 0)
    assert (d["t4_variant"] & 4 != 0) == (ldb % 8 != 0)
    assert_close_full(spec, x, got, 1e-2, kind="rel")


def test_matmul_bf16_full_size():
    spec = S.matmul(4096, 4096, 4096, "bf16")
    x = G.matmul_inputs(4096, 4096, 4096, "bf16", "signed")
    got, p = run_gpu(spec, x)
    assert p.template == "T4_tcgen05_contraction"
    assert_close_points(spec, x, got, 1e-2, n=3000, kind="scale")
    x = G.matmul_inputs(4096, 4096, 4096, "bf16", "ones")
    got, _ = run_gpu(spec, x)
    assert np.all(got[0] == 4096.0)
    x = G.matmul_inputs(4096, 4096, 4096, "bf16", "identity")
    got, _ = run_gpu(spec, x)
    assert np.array_equal(got[0], G.bf16_bits_to_f32(x[1]))


@pytest.mark.parametrize("M", [512, 1024, 2048])
@pytest.mark.parametrize("dt", ["bf16", "f32"])
def test_matmul_per_rank_shapes(M, dt):
    """The per-rank shapes of MatMul 4096³ sharded on M over 8 / 4 / 2 GPUs,
    each with the tiles the table holds for that bucket (bf16: stream-K narrow tiles at
    M = 512), on T4 (bf16) and T3 (fp32): sampled points against the oracle, plus the
    ones → K closed form."""
    spec = S.matmul(M, 4096, 4096, dt)
    x = G.matmul_inputs(M, 4096, 4096, dt, "signed")
    got, p = run_gpu(spec, x)
    assert p.template == ("T4_tcgen05_contraction" if dt == "bf16" else "T3_simt_contraction")
    assert_close_points(spec, x, got, 1e-2 if dt == "bf16" else 1e-4, n=4000, kind="scale")
    ones = G.matmul_inputs(M, 4096, 4096, dt, "ones")
    got, _ = run_gpu(spec, ones, plan=p)
    assert np.all(got[0] == 4096.0)


def test_ccsd_paper_inp1_full():
    """The paper's CCSD(T) Inp.1 reading (C-22) checked in FULL — every one of the 37.7 M
    outputs against the fp64 oracle — in fp32 (T3) and bf16 (T4)."""
    for dt, tol in (("f32", 1e-4), ("bf16", 1e-2)):
        spec = S.ccsd_sd2(dtype=dt)
        x = G.gen_inputs(spec, 4011)
        got, _ = run_gpu(spec, x)
        assert_close_full(spec, x, got, tol, kind="scale")


def test_ccsd_bf16_tcgen05():
    # tiny brute-force size, the paper's Inp.1 reading (C-22), then the O=24/V=72 config sampled
    for spec, n in ((S.ccsd_sd1(2, 3, "bf16"), None), (S.ccsd_sd2(dtype="bf16"), 20000),
                    (S.ccsd_sd1(24, 72, "bf16"), 20000)):
        x = G.gen_inputs(spec, 4010)
        got, p = run_gpu(spec, x)
        assert p.template == "T4_tcgen05_contraction"
        if n is None:
            assert_close_full(spec, x, got, 1e-2, kind="scale")
        else:
            assert_close_points(spec, x, got, 1e-2, n=n, kind="scale")


@pytest.mark.parametrize("cfg", [(2, 3, 4, 16, 3, 3, 8), (1, 7, 7, 512, 3, 3, 512), (1, 112, 112, 64, 7, 7, 3)])
def test_mcc_bf16_tcgen05(cfg):
    spec = S.mcc(*cfg, dtype="bf16")
    x = G.mcc_inputs(spec)
    got, p = run_gpu(spec, x)
    assert p.template == "T4_tcgen05_contraction"
    assert_close_full(spec, x, got, 1e-2, kind="scale")


@pytest.mark.parametrize("tile", ["implicit=1", "implicit=2", "implicit=3", "cluster=2"])
def test_t4_variants_parity(tile):
    """T4 A-operand variants on MCC (1: implicit-GEMM N-d TMA box, 2: in-kernel cp.async
    gather, 3: gather pre-pass) and 2-SM pairs on MatMul."""
    if tile.startswith("implicit"):
        spec = S.mcc(128, 7, 7, 128, 3, 3, 128, "bf16")
        x = G.mcc_inputs(spec)
        got, p = run_gpu(spec, x, force_tile=tile)
        v = p.describe()["t4_variant"]
        assert v & {"implicit=1": 16, "implicit=2": 32, "implicit=3": 2}[tile], v
        assert_close_points(spec, x, got, 1e-2, n=4000, kind="scale")
    else:
        spec = S.matmul(1024, 768, 640, "bf16")
        x = G.matmul_inputs(1024, 768, 640, "bf16", "positive")
        got, p = run_gpu(spec, x, force_tile=tile)
        assert p.describe()["t4_variant"] & 8
        assert_close_full(spec, x, got, 1e-2, kind="rel")


@pytest.mark.parametrize("shape,tile,out", [((2560, 2048, 1024), "cluster=1,split=3", "f32"),
                                            ((2500, 2000, 1000), "cluster=1,split=2", "f32"),
                                            ((2500, 2000, 1000), "split=4", "bf16")])
def test_t4_split_tail_1sm(shape, tile, out):
    """1-SM split-K tail: the partial last wave's tiles split along K (fused fixup in split
    order), row-major (EPI 0) and table-scatter bf16 (EPI 1) epilogues, ragged M/N/K."""
    M, N, K = shape
    spec = S.matmul(M, N, K, "bf16", out_dtype=out)
    x = G.matmul_inputs(M, N, K, "bf16", "positive")
    plan = None
    for _ in range(2):                      # second run: the tail counters were reset
        got, plan = run_gpu(spec, x, plan=plan, force_tile=tile)
        assert not plan.describe()["t4_variant"] & 8
        assert_close_points(spec, x, got, 1e-2, n=20000, kind="rel")


@pytest.mark.parametrize("shape,tile,kind", [((512, 512, 8192), "split=2", "full"),  # 4 tiles, ~16 pairs each
                                             ((2500, 2000, 1000), "bn=256,split=2", "points"),   # ragged, 80 tiles / 74 pairs
                                             ((4096, 4096, 4096), "bn=256,split=2", "points"),   # 3 whole waves + SK
                                             ((1024, 768, 640), "split=1", "full"),   # whole tiles only
                                             ((700, 1000, 1000), "cluster=4", "full"),  # odd row tiles: an idle pair
                                             ((2500, 2000, 1000), "cluster=4", "points"),  # 4-CTA clusters
                                             ((512, 768, 4096), "bn=512", "full"),    # wide 256x512 pair tiles
                                             ((2500, 2000, 1000), "bn=512", "points"),
                                             ((4096, 4096, 4096), "bn=512", "points")])
def test_t4_stream_k(shape, tile, kind):
    """2-SM stream-K hybrid (forced with split≥2 where the auto rule / tile table would pick
    whole tiles): whole-tile waves, then each cluster's even share of the remaining
    (tile, k-block) space; producers publish coalesced fp32 partials, the finisher (the one
    holding k = 0) adds them in k order.  Single pairs (default) and 4-CTA clusters
    (cluster=4: two pairs sharing B by TMA multicast; with an odd number of 256-row tiles
    the last pair computes zero-filled rows and stores nothing), and wide 256×512 pair
    tiles (bn=512: two N=256 MMAs per k-step, per-column-half accumulator release).  Run
    twice on one plan: the flags return to rest."""
    M, N, K = shape
    spec = S.matmul(M, N, K, "bf16")
    x = G.matmul_inputs(M, N, K, "bf16", "positive")
    plan = None
    first = None
    for _ in range(2):
        got, plan = run_gpu(spec, x, plan=plan, force_tile=tile)
        assert plan.describe()["t4_variant"] & 8
        if kind == "full":
            assert_close_full(spec, x, got, 1e-2, kind="rel")
        else:
            assert_close_points(spec, x, got, 1e-2, n=20000, kind="rel")
        if first is None:
            first = got[0].copy()
        else:
            assert np.array_equal(first, got[0])          # deterministic fixup order
    if shape == (4096, 4096, 4096):
        ones = G.matmul_inputs(M, N, K, "bf16", "ones")
        got, _ = run_gpu(spec, ones, plan=plan)
        assert np.all(got[0] == float(K))


@pytest.mark.parametrize("shape,bt,ns", [((4096, 4096, 4096), False, 1), ((512, 4096, 4096), False, 1),
                                         ((700, 1000, 1000), False, 1), ((300, 1000, 512), True, 1),
                                         ((12544, 512, 1024), False, 1), ((256, 384, 128), True, 1),
                                         ((4096, 4096, 4096), False, 2), ((2500, 4000, 256), False, 2),
                                         ((2560, 4096, 320), True, 2), ((2500, 3900, 200), True, 2)])
def test_t4_column_unit_stream(shape, bt, ns):
    """Wide 2-SM pair tiles under the column-unit stream schedule (tile knob nstream=1):
    every pair takes an equal share of 128-column units of 256-row strips, whole K, as
    tiles of 1-4 units (an odd last unit runs as an N = 128 MMA with 64 columns per CTA);
    nstream=2: whole tiles for the complete waves, units only in the partial last wave;
    ragged M / N, MN-major and K-major B; repeatable bit for bit."""
    M, N, K = shape
    spec = _mm_spec(M, N, K, False, bt)
    x = G.gen_inputs(spec, 3150, "positive")
    plan = None
    first = None
    for _ in range(2):
        got, plan = run_gpu(spec, x, plan=plan, force_tile=f"bn=512,nstream={ns},split=1")
        assert plan.describe()["t4_variant"] & 8
        if M * N <= 1000 * 1000:
            assert_close_full(spec, x, got, 1e-2, kind="rel")
        else:
            assert_close_points(spec, x, got, 1e-2, n=20000, kind="rel")
        if first is None:
            first = got[0].copy()
        else:
            assert np.array_equal(first, got[0])


@pytest.mark.parametrize("shape,out", [((100, 300, 4096), "f32"), ((100, 300, 4096), "bf16"), ((64, 512, 2048), "f32")])
def test_t4_few_tile_splitk(shape, out):
    """1-SM kernel with few tiles and a deep K (as MCC conv5_1 at N = 1): every tile is split
    along K over the idle SMs, all splits write partials, t4_xfold_kernel folds them in split
    order; ragged M / N, fp32 and bf16 outputs; deterministic across runs."""
    M, N, K = shape
    spec = S.matmul(M, N, K, "bf16", out_dtype=out)
    x = G.matmul_inputs(M, N, K, "bf16", "positive")
    got, p = run_gpu(spec, x)
    assert not p.describe()["t4_variant"] & 8
    assert_close_full(spec, x, got, 1e-2, kind="rel")
    got2, _ = run_gpu(spec, x, plan=p)
    assert np.array_equal(got[0], got2[0])


@pytest.mark.parametrize("cfg", [(1, 9, 13, 64, 7, 7, 3), (3, 17, 19, 64, 7, 7, 3), (2, 112, 112, 64, 7, 7, 3),
                                 (2, 20, 21, 64, 3, 3, 3)])
def test_mcc_small_k_direct(cfg):
    """MCC with C = 3 (conv1 7×7/s2, Fig 3 MCC Inp.2 P:529, reading C-21; and a 3×3 layer) on
    the small-K direct kernel (t4_conv.cu): A rows built in TMEM from staged input runs.
    Ragged last tiles (M = 117, 969) and tiles straddling two images (P·Q = 323) included;
    full comparison with the fp64 oracle on the same bf16 inputs."""
    spec = S.mcc(*cfg, dtype="bf16")
    x = G.mcc_inputs(spec)
    got, p = run_gpu(spec, x)
    assert p.template == "T4_tcgen05_contraction"
    assert p.describe()["t4_variant"] == 1024, p.describe()
    assert_close_full(spec, x, got, 1e-2, kind="scale")


def test_mcc_conv1_config_sampled():
    """conv1 7×7/s2 at N = 256 (C4b-B): 20 000 sampled outputs, each
    folded over its full 147-term window by the oracle; plus determinism (bit-identical rerun)."""
    spec = S.mcc(256, 112, 112, 64, 7, 7, 3, "bf16")
    x = G.mcc_inputs(spec)
    got, p = run_gpu(spec, x)
    assert p.describe()["t4_variant"] == 1024
    assert_close_points(spec, x, got, 1e-2, n=20000, kind="scale")
    got2, _ = run_gpu(spec, x, plan=p)
    assert np.array_equal(got[0], got2[0])


def test_mcc_bf16_config_sampled():
    spec = S.mcc(256, 7, 7, 512, 3, 3, 512, "bf16")
    x = G.mcc_inputs(spec)
    got, _ = run_gpu(spec, x)
    assert_close_points(spec, x, got, 1e-2, n=5000, kind="scale")


@pytest.mark.parametrize("case", ["bulk_ragged", "bulk_O4_V72", "run8_sd2", "run8_forced"])
def test_t4_scatter_epilogues(case):
    """T4 scatter epilogues on CCSD(T)-shaped outputs (orientation swapped so t3's unit-stride
    p4 is on the TMEM column axis): EPI 3 bulk runs (L = V, N-tile 2L; ragged M, a last
    N-tile holding one run, row pieces broken at h3 and tile edges), EPI 2 run-8 vectors
    (sd2: p4 runs of 16; sd1 with the bulk kernel disabled by tile knob epi=1)."""
    spec, tile, bit = {
        "bulk_ragged": (S.ccsd_sd1(3, 40, "bf16"), None, 128),
        "bulk_O4_V72": (S.ccsd_sd1(4, 72, "bf16"), None, 128),
        "run8_sd2": (S.ccsd_sd2(dtype="bf16"), None, 64),
        "run8_forced": (S.ccsd_sd1(3, 40, "bf16"), "epi=1", 64),
    }[case]
    x = G.gen_inputs(spec, 4020)
    got, p = run_gpu(spec, x, force_tile=tile)
    v = p.describe()["t4_variant"]
    assert v & bit, v
    if case == "bulk_O4_V72":
        assert_close_points(spec, x, got, 1e-2, n=50000, kind="scale")
    else:
        assert_close_full(spec, x, got, 1e-2, kind="scale")


# ------------------------------------------- F4: the remaining Fig 3 workloads (paper sizes)
PAPER_CASES = {
    # name: (spec builder, input seed, sampled points or None = full check)
    "matmul_1024": (lambda: S.matmul(1024, 1024, 1024, "f32"), 7001, 20000),
    "matmul_1x2048x1000": (lambda: S.matmul(1, 1000, 2048, "f32"), 7002, None),
    "matmul_t_10x500x64": (lambda: S.matmul_t(10, 500, 64, "f32"), 7003, None),
    "bmatmul_16x10x500x64": (lambda: S.bmatmul(16, 10, 500, 64, "f32"), 7004, None),
    "ccsd_inp1_sd2": (lambda: S.ccsd_sd2(), 7005, 20000),
    "ccsd_inp2_sd1x": (lambda: S.ccsd_sd1x(24, 16, 24, 16, 16, 24, 16), 7006, 20000),
    "mcc_caps_small": (lambda: S.mcc_caps(2, 5, 3, 4, 3, 3, 3), 7007, None),
    "mcc_caps_inp2": (lambda: S.mcc_caps(1, 112, 112, 64, 7, 7, 3), 7008, 5000),
    "mcc_caps_small_bf16": (lambda: S.mcc_caps(2, 5, 3, 4, 3, 3, 3, dtype="bf16"), 7009, None),
    "mcc_caps_inp2_bf16": (lambda: S.mcc_caps(1, 112, 112, 64, 7, 7, 3, dtype="bf16"), 7010, 5000),
}


@pytest.mark.parametrize("case", sorted(PAPER_CASES))
def test_fig3_paper_sizes(case):
    """MatMul (1024³; 1×2048 · 2048×1000), MatMul^T, bMatMul, CCSD(T) Inp.1/Inp.2 and MCC_Caps
    (Fig 3; readings C-22, C-33) through whatever template the planner picks."""
    build, seed, n = PAPER_CASES[case]
    spec = build()
    x = G.gen_inputs(spec, seed)
    got, p = run_gpu(spec, x)
    tol = 1e-2 if spec["inputs"][0]["dtype"] == "bf16" else 1e-4
    if n is None:
        assert_close_full(spec, x, got, tol, kind="scale")
    else:
        assert_close_points(spec, x, got, tol, n=n, kind="scale")


@pytest.mark.parametrize("cfg,tile", [((256, 7, 7, 512, 3, 3, 512), None),           # conv5_1, 2-SM
                                      ((3, 3, 5, 128, 3, 3, 64), None),              # P != Q, ragged M
                                      ((2, 9, 4, 256, 3, 3, 128), "cluster=1"),      # 1-SM kernel
                                      ((64, 7, 7, 512, 3, 3, 512), "bn=256"),        # narrow pair tiles, stream-K
                                      ((64, 7, 7, 512, 3, 3, 512), "split=1"),       # wide pair tiles, whole tiles
                                      ((3, 3, 5, 384, 3, 3, 64), "bn=512"),          # wide, ragged N
                                      ((5, 6, 6, 64, 2, 2, 64), None)])              # 2x2 window
def test_mcc_im2col_tma(cfg, tile):
    """T4 A operand through a TMA im2col map (window origin walk with traversal strides,
    filter taps as im2col offsets; no gather pre-pass, no gather warps)."""
    spec = S.mcc(*cfg, dtype="bf16")
    x = G.mcc_inputs(spec)
    got, p = run_gpu(spec, x, force_tile=tile)
    v = p.describe()["t4_variant"]
    assert v & 256, v
    if np.prod(cfg) > 1e9:
        assert_close_points(spec, x, got, 1e-2, n=20000, kind="scale")
    else:
        assert_close_full(spec, x, got, 1e-2, kind="scale")
