"""The NCCL data plane of the partitioner on ONE GPU: a one-rank plan with an
NCCL communicator (mdh_comm_init over a one-rank torch.distributed group) and an explicit
pw shard dim runs exactly the multi-GPU path of mdh_execute — local partial, then
ncclAllGather + the ordered ⊗ combine, or ncclAllReduce where ⊕ is exact in any order —
over a one-rank communicator.  (NCCL refuses two ranks on one device, so the ≥ 2-rank
exchange itself runs only on a multi-GPU box: bench.py --gpus N.)"""
import socket

import numpy as np
import pytest

import oracle
from gpu_util import assert_close_full, run_gpu
from mdh_workloads import gen as G
from mdh_workloads import specs as S

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def comm():
    import torch
    import torch.distributed as dist
    from paper_conf_sc_schulzegr25_b200 import Comm
    own = not dist.is_initialized()
    if own:
        s = socket.socket()
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
        s.close()
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1)
    c = Comm(device=torch.device("cuda", 0))
    yield c
    c.close()
    if own:
        dist.destroy_process_group()


def _plan(spec, comm, dim, flags=0):
    from paper_conf_sc_schulzegr25_b200 import Plan
    p = Plan(spec, world_size=1, rank=0, comm=comm, shard_dim=dim, flags=flags)
    d = p.describe()
    assert d["shard_is_red"] and d["shard_dim"] == dim, d
    return p


def test_nccl_allgather_ordered_combine_dot_f32(comm):
    """float pw(add): allgather + ordered combine (deterministic); bit-identical reruns."""
    spec = S.dot((1 << 20) + 3, "f32")
    x = G.dot_inputs((1 << 20) + 3, "f32", "positive")
    p = _plan(spec, comm, 0)
    got, _ = run_gpu(spec, x, plan=p)
    assert_close_full(spec, x, got, 1e-4, kind="rel")
    got2, _ = run_gpu(spec, x, plan=p)
    assert np.array_equal(got[0], got2[0])


def test_nccl_allreduce_int_wrap(comm):
    """int32 pw(add) (wrap mod 2^32, reading C-12): ncclAllReduce with ncclUint32, exact."""
    spec = S.dot(1 << 20, "i32")
    x = G.dot_inputs(1 << 20, "i32", "iota_iota")
    got, _ = run_gpu(spec, x, plan=_plan(spec, comm, 0))
    assert int(got[0][0]) == 1431830528                      # tests/golden/dot_int32.json
    assert_close_full(spec, x, got, 0, kind="exact")


@pytest.mark.parametrize("op", ["PW_PRL_ARGMAX", "PW_PRL_PAPER"])
def test_nccl_allgather_prl(op, comm):
    """custom PRL operators (NCCL cannot express them): allgather of the packed records,
    then the ordered combine kernel; bit-exact."""
    N, I = 700, 3000
    ins = G.prl_inputs(N, I, seed_base=5650)
    spec = S.prl(N, I, op)
    got, _ = run_gpu(spec, ins, plan=_plan(spec, comm, 1))
    assert_close_full(spec, ins, got, 0, kind="exact")


def test_nccl_float_allreduce_splitk(comm):
    """MatMul split along K through ncclAllReduce (MDH_PLAN_FLOAT_ALLREDUCE, F3)."""
    from paper_conf_sc_schulzegr25_b200 import FLOAT_ALLREDUCE
    spec = S.matmul(96, 80, 1000)
    x = G.matmul_inputs(96, 80, 1000, "f32", "positive")
    got, _ = run_gpu(spec, x, plan=_plan(spec, comm, 2, FLOAT_ALLREDUCE))
    assert_close_full(spec, x, got, 1e-4, kind="rel")


def test_nccl_allreduce_keeps_untouched_elements(comm):
    """int max over a strided output image (y[3i+1], 151 elements, 50 written): the
    allreduce runs in the workspace and only the image is placed (reading C-5)."""
    import torch
    from paper_conf_sc_schulzegr25_b200 import to_device, to_numpy
    d = ["i", "k"]
    spec = S.make_spec("strided_i32", d, [50, 30], ["CC", "PW_MAX"], "IDENTITY",
                       [S.buffer("x", "i32", [["i", "k"]], d)],
                       [S.buffer("y", "i32", [["3*i+1"]], d, shape=[151])])
    x = G.gen_inputs(spec, 2810)
    p = _plan(spec, comm, 1)
    y = torch.full((151,), -7, dtype=torch.int32, device="cuda")
    p([to_device(x[0], "i32", "cuda")], [y])
    torch.cuda.synchronize()
    ref = oracle.evaluate(spec, x)[0].astype(np.int64)
    got = to_numpy(y, "i32").astype(np.int64)
    img = np.zeros(151, bool)
    img[3 * np.arange(50) + 1] = True
    assert np.array_equal(got[img], ref[img])
    assert np.all(got[~img] == -7)
