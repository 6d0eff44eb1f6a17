"""mdh_execute_host's pipeline (include/mdh.h): the problem cut into 4 chunks along a cc
dim, chunk c's H2D copies, computation and D2H copies on three streams so both PCIe
directions overlap the kernels.  Each case runs through the C-ABI with pinned host
buffers and is compared with the CPU oracle (tolerances: DESIGN.md §5); the plan's
description names the chunk dim.  MDH_HOST_PIPE_MIN_MB=0 lets small problems pipeline."""
import numpy as np
import pytest

from mdh_workloads import gen as G
from mdh_workloads import specs as S

from gpu_util import assert_close_full

pytestmark = pytest.mark.gpu


def _run_host(spec, x, plan=None):
    import torch
    from paper_conf_sc_schulzegr25_b200 import Plan, to_numpy
    p = plan or Plan(spec)
    hin = []
    for a, b in zip(x, spec["inputs"]):
        a = np.ascontiguousarray(a)
        t = torch.from_numpy(a.view(np.int16) if b["dtype"] == "bf16" else a)
        hin.append(t.pin_memory())
    douts = p.empty_outputs(torch.device("cuda", 0))
    hout = [torch.empty(o.shape, dtype=o.dtype).pin_memory() for o in douts]
    for o in hout:
        o.view(torch.uint8).fill_(0x7F)
    n = p.host_scratch_bytes()
    scratch = torch.empty(n, dtype=torch.uint8, device="cuda")
    st = torch.cuda.current_stream()
    p.execute_host(hin, hout, scratch.data_ptr(), n, st.cuda_stream)
    torch.cuda.synchronize()
    return [to_numpy(o, b["dtype"]) for o, b in zip(hout, spec["outputs"])], p


CASES = {
    # MatMul rows (A and C sliced, B copied once); ragged row chunks
    "matmul_bf16": (lambda: S.matmul(1000, 768, 512, "bf16"), lambda sp: G.matmul_inputs(1000, 768, 512, "bf16", "positive"),
                    1e-2, "rel", 0),
    "matmul_f32": (lambda: S.matmul(600, 256, 300, "f32"), lambda sp: G.matmul_inputs(600, 256, 300, "f32", "positive"),
                   1e-4, "rel", 0),
    # Jacobi planes: overlapping input slabs (halo planes), interior output planes
    "jacobi3d": (lambda: S.jacobi3d(34, 40, 44), lambda sp: G.jacobi3d_inputs(34, 40, 44), 1e-4, "scale", 0),
    # MCC images on n (im2col A through TMA per chunk)
    "mcc_bf16": (lambda: S.mcc(8, 7, 7, 64, 3, 3, 32, "bf16"), lambda sp: G.mcc_inputs(sp), 1e-2, "scale", 0),
    # PRL new records on n (17 input buffers, 3 outputs; DB fields copied once): bit-exact
    "prl": (lambda: S.prl(4096, 1024), lambda sp: G.prl_inputs(4096, 1024), 0, "exact", 0),
}


@pytest.mark.parametrize("name", list(CASES))
def test_host_pipeline(name, monkeypatch):
    monkeypatch.setenv("MDH_HOST_PIPE_MIN_MB", "0")
    mk, inp, tol, kind, dim = CASES[name]
    spec = mk()
    x = inp(spec)
    got, p = _run_host(spec, x)
    d = p.describe()
    assert "host_pipe" in d and d["host_pipe"]["chunks"] == 4 and d["host_pipe"]["dim"] == dim, d.get("host_pipe")
    assert_close_full(spec, x, got, tol, kind=kind)
    got2, _ = _run_host(spec, x, plan=p)              # the plan's streams and sub-plans are reused
    for a, b in zip(got, got2):
        assert np.array_equal(a, b)


def test_host_pipeline_off_and_fallback(monkeypatch):
    """MDH_HOST_PIPE=0 keeps the one-shot path; a problem below the size threshold too; both
    give the oracle's result."""
    monkeypatch.setenv("MDH_HOST_PIPE", "0")
    spec = S.matmul(600, 256, 300, "f32")
    x = G.matmul_inputs(600, 256, 300, "f32", "positive")
    got, p = _run_host(spec, x)
    assert "host_pipe" not in p.describe()
    assert_close_full(spec, x, got, 1e-4, kind="rel")
    monkeypatch.delenv("MDH_HOST_PIPE")
    got, p = _run_host(spec, x)                       # 1.9 MB < 32 MB: not pipelined
    assert "host_pipe" not in p.describe()
    assert_close_full(spec, x, got, 1e-4, kind="rel")
