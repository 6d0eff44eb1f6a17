"""N>1 host-side logic on CPU: two processes (gloo, world_size 2 and 3) each plan their
sub-domain with libmdh (world_size>1, no GPU needed to plan), evaluate it with the CPU
oracle on the slices `mdh_plan_local_shape` reports, exchange results over
torch.distributed, and rank 0 reassembles — concatenation for a cc shard, ordered ⊗ in
rank order for a pw shard — and compares with the unsharded oracle.
This pins the partitioner (sub-domain rewrite, local origins, halo planes, rank order)
independently of the GPU."""
import copy
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def local_spec(spec, d, start, length, shapes_offsets):
    """Test-side restatement of the sub-domain rewrite: size[d] := length; every access
    offset += coeff[:, d]·start (outputs only for a cc dim), then minus the local origin."""
    s = copy.deepcopy(spec)
    s["sizes"][d] = length
    nin = len(spec["inputs"])
    for b, buf in enumerate(s["inputs"] + s["outputs"]):
        shp, off = shapes_offsets[b]
        buf["shape"] = list(shp)
        is_out = b >= nin
        for acc in buf["acc"]:
            for r in range(len(acc["offset"])):
                if not (is_out and spec["ops"][d] != "CC"):
                    acc["offset"][r] += acc["coeff"][r][d] * start
                acc["offset"][r] -= off[r]
    return s


def _worker(rank, world, port, name, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import sys
    sys.path.insert(0, ROOT)
    import oracle
    from mdh_workloads import gen as G
    from mdh_workloads import specs as S
    from paper_conf_sc_schulzegr25_b200 import Plan, VIRTUAL_SHARD
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        if name == "matmul":
            spec, ins = S.matmul(37, 20, 11), G.matmul_inputs(37, 20, 11, "f32", "positive")
        elif name == "jacobi3d":
            spec, ins = S.jacobi3d(13, 6, 7), G.jacobi3d_inputs(13, 6, 7)
        elif name == "dot_i32":
            spec, ins = S.dot(1001, "i32"), G.dot_inputs(1001, "i32")
        elif name == "prl_paper":
            spec, ins = S.prl(30, 257, "PW_PRL_PAPER"), G.prl_inputs(30, 257, seed_base=5700)
        else:
            spec, ins = S.prl(30, 257), G.prl_inputs(30, 257, seed_base=5700)
        p = Plan(spec, world_size=world, rank=rank, flags=VIRTUAL_SHARD)
        desc = p.describe()
        d, start, length = desc["shard_dim"], desc["shard_start"], desc["shard_len"]
        so = [p.local_shape(False, b)[:2] for b in range(len(spec["inputs"]))]
        so += [p.local_shape(True, b)[:2] for b in range(len(spec["outputs"]))]
        lins = []
        for b, x in enumerate(ins):
            shp, off = so[b]
            lins.append(np.ascontiguousarray(x[tuple(slice(o, o + s) for o, s in zip(off, shp))]))
        lspec = local_spec(spec, d, start, length, so)
        louts = oracle.evaluate(lspec, lins)
        gathered = [None] * world
        dist.all_gather_object(gathered, (desc, so, louts))
        if rank == 0:
            full = oracle.evaluate(spec, ins)
            nin = len(spec["inputs"])
            if not desc["shard_is_red"]:
                covered = [np.zeros(o.shape, bool) for o in full]
                for gd, gso, go in gathered:
                    for b, o in enumerate(go):
                        shp, off = gso[nin + b]
                        sl = tuple(slice(a, a + s) for a, s in zip(off, shp))
                        assert np.array_equal(o, full[b][sl]), f"{name}: shard mismatch"
                        assert not covered[b][sl].any(), "overlapping shards"
                        covered[b][sl] = True
                assert all(c.all() for c in covered), "shards do not cover the output"
            else:
                acc = gathered[0][2]
                for gd, gso, go in gathered[1:]:
                    if spec["f"] == "PRL_COMPARE":
                        paper = spec["ops"][1] == "PW_PRL_PAPER"
                        li, lw, lm = acc
                        ri, rw, rm = go
                        if paper:
                            take_l = (lm == 14) & (rm != 14)
                        else:
                            kl = np.stack([(lm == 14), lw, li.astype(np.float64)], 0)
                            kr = np.stack([(rm == 14), rw, ri.astype(np.float64)], 0)
                            take_l = np.ones(li.shape, bool)
                            dec = np.zeros(li.shape, bool)
                            for c in range(3):
                                gt = (kr[c] > kl[c]) & ~dec
                                lt = (kr[c] < kl[c]) & ~dec
                                take_l[gt] = False
                                dec |= gt | lt
                        acc = [np.where(take_l, a, b) for a, b in zip(acc, go)]
                    else:   # int32 wrap add
                        acc = [((a.astype(np.int64) + b.astype(np.int64)) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
                               for a, b in zip(acc, go)]
                for a, f in zip(acc, full):
                    assert np.array_equal(a, f), f"{name}: combined pw shards differ"
            starts = [g[0]["shard_start"] for g in gathered]
            assert starts == sorted(starts), "rank order must be index order"
            q.put("ok")
    except Exception as e:  # report to the parent
        q.put(f"rank {rank}: {type(e).__name__}: {e}")
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("name", ["matmul", "jacobi3d", "dot_i32", "prl_argmax", "prl_paper"])
def test_sharded_plans_reassemble(name, world):
    from paper_conf_sc_schulzegr25_b200 import build
    build.build()
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(180)
    msgs = []
    while not q.empty():
        msgs.append(q.get())
    assert all(pr.exitcode == 0 for pr in procs), msgs
    assert "ok" in msgs, msgs


def _sweeps_worker(rank, world, port, q):
    """One z-slab of a Jacobi_3D time-stepping run (reading C-34): the rank's slab with one
    halo plane per side, swept by the oracle, and after every sweep the exchange
    mdh_stencil_sweeps performs — first owned plane (1) to rank-1's top halo, last owned
    plane (nz-2) to rank+1's bottom halo — over torch.distributed point-to-point."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import sys
    sys.path.insert(0, ROOT)
    import torch
    import oracle
    from mdh_workloads import specs as S
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        Z, Y, X, T = 11, 6, 7, 4
        u0 = np.random.Generator(np.random.PCG64(3402)).random((Z, Y, X)).astype(np.float32)
        lo, hi = S.z_slabs(Z, world)[rank]
        nz = hi - lo + 2
        spec = S.jacobi3d_sweep(nz, Y, X)
        u = u0[lo - 1:hi + 1].astype(np.float64)
        for _ in range(T):
            u = oracle.stencil_sweeps(spec, u, 1)
            t = torch.from_numpy(u)
            reqs = []
            if rank > 0:
                reqs.append(dist.isend(t[1].contiguous(), rank - 1))
                lo_recv = torch.empty_like(t[0])
                reqs.append(dist.irecv(lo_recv, rank - 1))
            if rank < world - 1:
                reqs.append(dist.isend(t[nz - 2].contiguous(), rank + 1))
                hi_recv = torch.empty_like(t[0])
                reqs.append(dist.irecv(hi_recv, rank + 1))
            for r in reqs:
                r.wait()
            if rank > 0:
                u[0] = lo_recv.numpy()
            if rank < world - 1:
                u[nz - 1] = hi_recv.numpy()
        gathered = [None] * world
        dist.all_gather_object(gathered, (lo, hi, u[1:nz - 1]))
        if rank == 0:
            full = oracle.stencil_sweeps(S.jacobi3d_sweep(Z, Y, X), u0, T)
            for glo, ghi, owned in gathered:
                assert np.array_equal(owned, full[glo:ghi]), f"slab [{glo},{ghi}) differs"
            q.put("ok")
    except Exception as e:
        q.put(f"rank {rank}: {type(e).__name__}: {e}")
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_stencil_sweeps_halo_exchange(world):
    """F3: z-sharded Jacobi_3D time-stepping with a per-sweep halo exchange
    reproduces the unsharded sweeps bit for bit (both fp64 oracle evaluations)."""
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    port = _free_port()
    procs = [ctx.Process(target=_sweeps_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(180)
    msgs = []
    while not q.empty():
        msgs.append(q.get())
    assert all(pr.exitcode == 0 for pr in procs), msgs
    assert "ok" in msgs, msgs
