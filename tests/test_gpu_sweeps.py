"""F3: stencil time-stepping through mdh_stencil_sweeps — the Jacobi_3D sweep
(reading C-34) applied T times, whole domain and z-sharded into slabs whose halo planes are
exchanged after every sweep (peer transport, virtual ranks on one GPU in lock-step)."""
import numpy as np
import pytest

import oracle
from mdh_workloads import specs as S

pytestmark = pytest.mark.gpu


def _ref(Z, Y, X, u0, T):
    sp = S.jacobi3d_sweep(Z, Y, X)
    ref = oracle.stencil_sweeps(sp, u0, T)
    sa = dict(sp, fparams=[abs(w) for w in sp["fparams"]])
    scale = oracle.stencil_sweeps(sa, np.abs(u0), T)
    return ref, scale


def _field(Z, Y, X, seed):
    return np.random.Generator(np.random.PCG64(seed)).random((Z, Y, X)).astype(np.float32) * 2 - 0.5


@pytest.mark.parametrize("zyx,T", [((34, 20, 37), 1), ((34, 20, 37), 4), ((9, 8, 131), 3), ((64, 64, 64), 5)])
def test_sweeps_whole_domain(zyx, T):
    import torch
    from paper_conf_sc_schulzegr25_b200 import Plan
    Z, Y, X = zyx
    u0 = _field(Z, Y, X, 3410 + Z)
    p = Plan(S.jacobi3d_sweep(Z, Y, X))
    u = torch.from_numpy(u0).cuda()
    v = u.clone()                                    # the fixed boundary shell lives in both
    res = p.stencil_sweeps(u, v, T)
    torch.cuda.synchronize()
    assert (res is v) == (T % 2 == 1)
    got = res.cpu().numpy().astype(np.float64)
    ref, scale = _ref(Z, Y, X, u0, T)
    assert np.array_equal(got[0], u0[0]) and np.array_equal(got[:, 0], u0[:, 0])   # boundary untouched
    err = np.abs(got - ref) / np.maximum(scale, 1e-30)
    assert err.max() <= 1e-4, err.max()


@pytest.mark.parametrize("Z,world", [(23, 2), (23, 3), (23, 5), (7, 5), (5, 3)])
def test_sweeps_zsharded_virtual_ranks(Z, world):
    """Slabs with one halo plane per side, a sweep per call in lock-step on one stream; after
    each sweep a rank's first / last owned plane is copied into the neighbours' halo planes
    (mdh_halo peer transport).  The owned planes equal the whole-domain GPU run bit for bit
    (same per-point arithmetic) and the fp64 oracle within the scale-normalised 1e-4.  The
    7-point kernel stores its first / last plane into the neighbours' halos itself (one
    launch per sweep).  Z = 7 / 5 give one-plane slabs (nz = 3) at every rank, rank 0 and
    the last rank included, whose single plane feeds one or both neighbours."""
    import torch
    from paper_conf_sc_schulzegr25_b200 import Halo, Plan
    Y, X, T = 12, 40, 4
    u0 = _field(Z, Y, X, 3420)
    whole = Plan(S.jacobi3d_sweep(Z, Y, X))
    wu = torch.from_numpy(u0).cuda()
    wres = whole.stencil_sweeps(wu, wu.clone(), T)
    slabs = S.z_slabs(Z, world)
    bufs, plans = [], []
    for lo, hi in slabs:
        b0 = torch.from_numpy(np.ascontiguousarray(u0[lo - 1:hi + 1])).cuda()
        bufs.append([b0, b0.clone()])
        plans.append(Plan(S.jacobi3d_sweep(hi - lo + 2, Y, X)))
    plane = Y * X * 4
    for t in range(T):
        s, d = t & 1, (t & 1) ^ 1
        for r, (lo, hi) in enumerate(slabs):
            h = Halo()
            h.rank, h.world = r, world
            order = (s, d)                           # this call's (u, v) = (src, dst)
            if r > 0:
                nzl = slabs[r - 1][1] - slabs[r - 1][0] + 2
                for k, i in enumerate(order):
                    h.peer_lo[k] = bufs[r - 1][i].data_ptr() + (nzl - 1) * plane
            if r < world - 1:
                for k, i in enumerate(order):
                    h.peer_hi[k] = bufs[r + 1][i].data_ptr()
            out = plans[r].stencil_sweeps(bufs[r][s], bufs[r][d], 1, halo=h)
            assert out is bufs[r][d]
            assert Plan.last_launch_count() == 1       # halo stores fused into the sweep kernel
    torch.cuda.synchronize()
    whole_np = wres.cpu().numpy()
    ref, scale = _ref(Z, Y, X, u0, T)
    fin = T & 1
    for r, (lo, hi) in enumerate(slabs):
        owned = bufs[r][fin].cpu().numpy()[1:hi - lo + 1]
        assert np.array_equal(owned, whole_np[lo:hi]), f"rank {r}: differs from the whole-domain run"
        err = np.abs(owned.astype(np.float64) - ref[lo:hi]) / np.maximum(scale[lo:hi], 1e-30)
        assert err.max() <= 1e-4


def test_sweeps_rejects_bad_plans():
    import torch
    from paper_conf_sc_schulzegr25_b200 import Halo, MdhError, Plan
    p = Plan(S.jacobi3d(10, 10, 10))                 # output 8³ ≠ input 10³
    u = torch.zeros(10, 10, 10, device="cuda")
    with pytest.raises(MdhError):
        p.stencil_sweeps(u, torch.zeros(8, 8, 8, device="cuda"), 1)
    q = Plan(S.jacobi3d_sweep(10, 10, 10))
    h = Halo()
    h.rank, h.world = 1, 2                           # no transport given
    with pytest.raises(MdhError):
        q.stencil_sweeps(u, u.clone(), 1, halo=h)
    with pytest.raises(MdhError):                    # u is v: aliasing (reading C-27)
        q.stencil_sweeps(u, u, 1)


def _box3_sweep(Y, X):
    """A 2-D 3×3 same-shape stencil sweep (v[i+1, j+1] = Σ w_rs·u[i+r, j+s], boundary ring
    kept) — runs on the box-window kernel, so the peer transport falls back to copies."""
    d = ["i", "j"]
    accs = [[f"i+{r}", f"j+{c}"] for r in range(3) for c in range(3)]
    wts = [0.05, 0.1, 0.05, 0.1, 0.3, 0.1, 0.05, 0.1, 0.05]
    return S.make_spec("box3_sweep", d, [Y - 2, X - 2], ["CC", "CC"], "STENCIL",
                       [S.buffer("u", "f32", accs, d, shape=[Y, X])],
                       [S.buffer("v", "f32", [["i+1", "j+1"]], d, shape=[Y, X])], fparams=wts)


@pytest.mark.parametrize("world", [1, 3])
def test_sweeps_box2d_copy_transport(world):
    """Non-7-point stencil: the sweep kernel cannot store halos itself, so after each sweep
    the boundary rows are copied into the neighbours' halo rows (device-to-device)."""
    import torch
    from paper_conf_sc_schulzegr25_b200 import Halo, Plan
    Y, X, T = 29, 68, 3
    u0 = _field(1, Y, X, 3430)[0]
    sp = _box3_sweep(Y, X)
    ref = oracle.stencil_sweeps(sp, u0, T)
    slabs = S.z_slabs(Y, world)
    bufs, plans = [], []
    for lo, hi in slabs:
        b0 = torch.from_numpy(np.ascontiguousarray(u0[lo - 1:hi + 1])).cuda()
        bufs.append([b0, b0.clone()])
        plans.append(Plan(_box3_sweep(hi - lo + 2, X)))
    row = X * 4
    for t in range(T):
        s, d = t & 1, (t & 1) ^ 1
        for r, (lo, hi) in enumerate(slabs):
            h = Halo()
            h.rank, h.world = r, world
            if r > 0:
                nzl = slabs[r - 1][1] - slabs[r - 1][0] + 2
                for k, i in enumerate((s, d)):
                    h.peer_lo[k] = bufs[r - 1][i].data_ptr() + (nzl - 1) * row
            if r < world - 1:
                for k, i in enumerate((s, d)):
                    h.peer_hi[k] = bufs[r + 1][i].data_ptr()
            plans[r].stencil_sweeps(bufs[r][s], bufs[r][d], 1, halo=h if world > 1 else None)
    torch.cuda.synchronize()
    for r, (lo, hi) in enumerate(slabs):
        owned = bufs[r][T & 1].cpu().numpy()[1:hi - lo + 1].astype(np.float64)
        assert np.max(np.abs(owned - ref[lo:hi])) <= 1e-5 * max(1.0, np.abs(ref).max())

