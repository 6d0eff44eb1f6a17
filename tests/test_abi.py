"""C-ABI checks that need no GPU: libmdh loads, exports every function include/mdh.h
declares, and mdh_plan validates specs / classifies dims / rewrites shards on the host
(SURVEY §8(b) conventions; readings C-3, C-5, C-8, C-9, C-10, C-27)."""
import ctypes
import os
import re

import pytest

from mdh_workloads import specs as S

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def mdh():
    from paper_conf_sc_schulzegr25_b200 import build
    build.build()
    import paper_conf_sc_schulzegr25_b200 as m
    return m


def header_functions():
    text = open(os.path.join(ROOT, "include", "mdh.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(mdh_[a-z_0-9]+)\s*\(", text)))


def test_library_exports_every_header_symbol(mdh):
    names = header_functions()
    assert len(names) >= 15
    L = ctypes.CDLL(mdh.library_path())
    for n in names:
        assert hasattr(L, n), n
    assert mdh.abi_version() == 3


def plan_status(mdh, spec, **kw):
    try:
        mdh.Plan(spec, **kw)
        return "OK"
    except mdh.MdhError as e:
        return e.status


def test_config_templates(mdh):
    cases = {
        "T2_reduce": [S.dot(1 << 20, "f32"), S.dot(1 << 20, "i32"), S.matvec(4096, 4096)],
        "T3_simt_contraction": [S.matmul(4096, 4096, 4096), S.ccsd_sd1(24, 72, "f32"),
                                S.mcc(256, 7, 7, 512, 3, 3, 512, "f32")],
        "T1_stencil": [S.jacobi3d(512, 512, 512), S.jacobi1d(1000)],
        "T5_prl_pairwise": [S.prl(1 << 20, 1 << 14), S.prl(1 << 14, 1 << 20, "PW_PRL_PAPER")],
    }
    for tmpl, specs in cases.items():
        for sp in specs:
            d = mdh.Plan(sp).describe()
            assert d["template"] == tmpl, (sp["name"], d)


def test_contraction_grouping(mdh):
    # t3's unit-stride p4 is a t2 dim, so the groups swap: N = {p4,h1,h2} (t2), M = {h3,p6,p5}
    d = mdh.Plan(S.ccsd_sd1(24, 72, "f32")).describe()["contraction"]
    assert (d["M"], d["N"], d["K"], d["Z"]) == (24 * 72 * 72, 72 * 24 * 24, 72, 1)
    d = mdh.Plan(S.mcc(256, 7, 7, 512, 3, 3, 512, "f32")).describe()["contraction"]
    assert (d["M"], d["N"], d["K"]) == (256 * 49, 512, 4608)
    d = mdh.Plan(S.bmatmul(16, 10, 500, 64)).describe()["contraction"]
    assert (d["Z"], d["M"], d["N"], d["K"]) == (16, 10, 500, 64)


def test_invalid_specs(mdh):
    d = ["i"]
    neg = S.make_spec("neg", d, [4], ["CC"], "IDENTITY", [S.buffer("x", "f32", [["i-1"]], d)],
                      [S.buffer("y", "f32", [["i"]], d)])
    assert plan_status(mdh, neg) == "INVALID_SPEC"
    small = S.make_spec("small", d, [4], ["CC"], "IDENTITY", [S.buffer("x", "f32", [["i"]], d, shape=[3])],
                        [S.buffer("y", "f32", [["i"]], d)])
    assert plan_status(mdh, small) == "INVALID_SPEC"
    zero = S.dot(5)
    zero["sizes"] = [0]
    assert plan_status(mdh, zero) == "INVALID_SPEC"                      # C-10
    nonin = S.make_spec("nonin", ["i", "j"], [3, 3], ["CC", "CC"], "IDENTITY",
                        [S.buffer("x", "f32", [["i", "j"]], ["i", "j"])], [S.buffer("y", "f32", [["i+j"]], ["i", "j"])])
    assert plan_status(mdh, nonin) == "INVALID_SPEC"                     # C-5
    ignore = S.make_spec("ign", ["i", "j"], [3, 3], ["CC", "CC"], "IDENTITY",
                         [S.buffer("x", "f32", [["i", "j"]], ["i", "j"])], [S.buffer("y", "f32", [["i"]], ["i", "j"])])
    assert plan_status(mdh, ignore) == "INVALID_SPEC"
    mixed = S.make_spec("mixed", ["a", "b"], [2, 2], ["PW_MAX", "PW_ADD"], "IDENTITY",
                        [S.buffer("x", "f32", [["a", "b"]], ["a", "b"])], [S.buffer("y", "f32", [["0"]], ["a", "b"], shape=[1])])
    assert plan_status(mdh, mixed) == "UNSUPPORTED"                      # C-3
    arity = S.dot(8)
    arity["inputs"] = arity["inputs"][:1]
    assert plan_status(mdh, arity) == "INVALID_SPEC"
    mixdt = S.dot(8)
    mixdt["inputs"][1]["dtype"] = "i32"
    assert plan_status(mdh, mixdt) == "UNSUPPORTED"
    prl_on_add = S.dot(8)
    prl_on_add["ops"] = ["PW_PRL_ARGMAX"]
    assert plan_status(mdh, prl_on_add) == "UNSUPPORTED"
    ok_strided = S.make_spec("str", d, [5], ["CC"], "IDENTITY", [S.buffer("x", "f32", [["i"]], d)],
                             [S.buffer("y", "f32", [["2*i"]], d, shape=[10])])
    assert plan_status(mdh, ok_strided) == "OK"


def test_shape_inference_and_declared(mdh):
    p = mdh.Plan(S.mcc(2, 3, 4, 5, 3, 3, 2, "f32"))
    assert p.in_shapes[0] == [2, 2 * 3 + 3 - 1, 2 * 4 + 3 - 1, 2]       # declared
    assert p.in_shapes[1] == [5, 3, 3, 2]                               # inferred (fn.7 P:316)
    assert p.out_shapes[0] == [2, 3, 4, 5]


def test_shard_rewrite_local_shapes(mdh):
    # MatMul sharded on M over 3 ranks: A and C rows split, B replicated
    sp = S.matmul(10, 6, 4)
    got = []
    for r in range(3):
        p = mdh.Plan(sp, world_size=3, rank=r, shard_dim=0, flags=mdh.VIRTUAL_SHARD)
        a, aoff, _ = p.local_shape(False, 0)
        b, boff, _ = p.local_shape(False, 1)
        c, coff, _ = p.local_shape(True, 0)
        got.append((a, aoff, b, boff, c, coff))
    assert [g[0][0] for g in got] == [4, 3, 3] and [g[1][0] for g in got] == [0, 4, 7]
    assert all(g[2] == [4, 6] and g[3] == [0, 0] for g in got)
    assert [g[4][0] for g in got] == [4, 3, 3]
    # Jacobi3D z-shard: each input slab carries the two halo planes
    sp = S.jacobi3d(20, 8, 8)
    for r in range(4):
        p = mdh.Plan(sp, world_size=4, rank=r, shard_dim=0, flags=mdh.VIRTUAL_SHARD)
        u, uoff, _ = p.local_shape(False, 0)
        v, voff, _ = p.local_shape(True, 0)
        assert u[0] == v[0] + 2 and uoff[0] == voff[0]
    # PRL DB-dim shard: outputs full, DB slices in rank order
    sp = S.prl(100, 1001)
    offs = []
    for r in range(4):
        p = mdh.Plan(sp, world_size=4, rank=r, flags=mdh.VIRTUAL_SHARD)
        d = p.describe()
        assert d["shard_dim"] == 1 and d["shard_is_red"]
        shp, off, _ = p.local_shape(False, 8)
        offs.append((off[0], shp[0]))
        assert p.local_shape(True, 0)[0] == [100]
    assert offs == [(0, 251), (251, 250), (501, 250), (751, 250)]


def test_pw_shard_without_comm_rejected(mdh):
    assert plan_status(mdh, S.prl(10, 100), world_size=2, rank=0) == "INVALID_ARG"


def test_tile_override_and_table(mdh, tmp_path):
    p = mdh.Plan(S.dot(1 << 20, "f32"), force_tile="split=7")
    assert p.describe()["tiles"]["split"] == 7
    t = tmp_path / "t.json"
    t.write_text('{"entries": [{"template": "T2_reduce", "dtype": "f32", "bucket": [0, 20], "tiles": {"split": 33}}]}')
    d = mdh.Plan(S.dot(1 << 20, "f32"), tile_table=str(t)).describe()
    assert d["tiles"]["split"] == 33 and d["tiles"]["source"].startswith("table")
    d = mdh.Plan(S.dot(1 << 22, "f32"), tile_table=str(t)).describe()   # nearest bucket
    assert d["tiles"]["split"] == 33
    # the key includes f and the ⊗-class when an entry records them
    t.write_text('{"entries": [{"template": "T2_reduce", "dtype": "f32", "f": "MUL", "op": "PW_MAX", '
                 '"bucket": [0, 20], "tiles": {"split": 44}}]}')
    assert mdh.Plan(S.dot(1 << 20, "f32", "PW_MAX"), tile_table=str(t)).describe()["tiles"]["split"] == 44
    assert mdh.Plan(S.dot(1 << 20, "f32"), tile_table=str(t)).describe()["tiles"]["source"] == "default"


def test_sweeps_argument_checks_on_host(mdh):
    """mdh_stencil_sweeps validates its pointers before enqueueing anything (no GPU needed):
    u == v or overlapping u/v (reading C-27), a pointer that is not 16-byte aligned, and
    the peer transport asked for more than one sweep per call (it has no cross-rank wait)
    are INVALID_ARG."""
    q = mdh.Plan(S.jacobi3d_sweep(10, 10, 10))
    L = mdh.lib()
    n = 10 * 10 * 10 * 4
    base = 1 << 32

    def call(u, v, sweeps=1, halo=None):
        res = ctypes.c_int32()
        return L.mdh_stencil_sweeps(q._h, u, v, sweeps, ctypes.byref(halo) if halo else None,
                                    None, 0, None, ctypes.byref(res))

    INVALID_ARG = 1
    assert call(base, base) == INVALID_ARG                       # u is v
    assert call(base, base + n // 2) == INVALID_ARG              # overlap
    assert call(base + 4, base + 2 * n) == INVALID_ARG           # misaligned u
    assert call(base, base + 2 * n + 8) == INVALID_ARG           # misaligned v
    h = mdh.Halo()
    h.rank, h.world = 0, 2
    h.peer_hi[0], h.peer_hi[1] = base + 8 * n, base + 9 * n
    assert call(base, base + 2 * n, sweeps=2, halo=h) == INVALID_ARG   # peer: one sweep per call
    h.peer_hi[1] = base + n                                      # a "peer" plane inside own v
    assert call(base, base + n, sweeps=1, halo=h) == INVALID_ARG


def test_tile_table_picks_the_matvec_row_range_mode(mdh):
    """The measured tile table (compiled in) selects T2's row-range kernel for MatVec 8192²
    and keeps warp mode for 4096² (tools/sweep_tiles.py, profiles/r2_matvec_jacobi_floor.txt);
    a forced mode=3 on a shape it cannot serve (row length not 1024·2^k) stays in warp mode."""
    d = mdh.Plan(S.matvec(8192, 8192)).describe()
    assert d["tiles"]["mode"] == 3 and "row-range" in d["why"], d
    d = mdh.Plan(S.matvec(4096, 4096)).describe()
    assert d["tiles"]["mode"] != 3 and "row-range" not in d["why"], d
    d = mdh.Plan(S.matvec(8192, 5000), force_tile="mode=3").describe()
    assert "row-range" not in d["why"], d
