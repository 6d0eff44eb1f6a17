"""Helpers for the GPU parity tests: run a spec through the C-ABI (libmdh) and compare
with the CPU oracle on the same seeded inputs (tolerances: DESIGN.md §5)."""
from __future__ import annotations

import copy

import numpy as np

import oracle
from mdh_workloads import gen as G

FLOAT = ("bf16", "f32", "f64")


def dev():
    import torch
    return torch.device("cuda", 0)


def run_gpu(spec, inputs, plan=None, fill=True, **plan_kw):
    """Execute `spec` on cuda:0 through mdh_execute; outputs are pre-filled with NaN /
    0x7F.. so that reading untouched memory or accumulating into it shows up."""
    import torch
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device, to_numpy
    p = plan or Plan(spec, **plan_kw)
    d = dev()
    tin = [to_device(x, b["dtype"], d) for x, b in zip(inputs, spec["inputs"])]
    outs = p.empty_outputs(d)
    if fill:
        for o in outs:
            if o.dtype.is_floating_point:
                o.fill_(float("nan"))
            else:
                o.view(torch.uint8).fill_(0x7F)
    p(tin, outs)
    torch.cuda.synchronize()
    return [to_numpy(o, b["dtype"]) for o, b in zip(outs, spec["outputs"])], p


def abs_spec_inputs(spec, inputs):
    """The scale S of reading C-14: the same computation on |terms| (|inputs|, |weights|)."""
    s2 = copy.deepcopy(spec)
    s2["fparams"] = [abs(w) for w in spec.get("fparams", [])]
    ins = []
    for x, b in zip(inputs, spec["inputs"]):
        if b["dtype"] == "bf16":
            ins.append((x & np.uint16(0x7FFF)).astype(np.uint16))
        elif b["dtype"] in FLOAT or b["dtype"] == "i32":
            ins.append(np.abs(x))
        else:
            ins.append(x)
    return s2, ins


def assert_close_full(spec, inputs, got, tol, kind="scale"):
    """Compare every output element with the full oracle.  kind: 'exact' (integers and
    selections), 'rel' (element-wise relative, positive data), 'scale' (|g-o|/S)."""
    ref = oracle.evaluate(spec, inputs)
    if kind == "scale":
        s2, ins2 = abs_spec_inputs(spec, inputs)
        scale = oracle.evaluate(s2, ins2)
    for b, (g, o) in enumerate(zip(got, ref)):
        g = np.asarray(g)
        if spec["outputs"][b]["dtype"] not in FLOAT or kind == "exact":
            assert np.array_equal(g.astype(o.dtype) if g.dtype != o.dtype else g, o), \
                f"output {b}: {np.count_nonzero(g != o)} mismatches"
            continue
        g64 = g.astype(np.float64) if spec["outputs"][b]["dtype"] != "bf16" else G.bf16_bits_to_f32(g).astype(np.float64)
        assert not np.any(np.isnan(g64)), "NaN in output (uncovered element or read of output)"
        err = np.abs(g64 - o)
        if kind == "rel":
            rel = err / np.maximum(np.abs(o), 1e-300)
            assert rel.max() <= tol, f"max rel err {rel.max():.3e} > {tol}"
        else:
            rel = err / np.maximum(np.abs(scale[b]), 1e-300)
            assert rel.max() <= tol, f"max scale-normalised err {rel.max():.3e} > {tol}"
    return ref


def assert_close_points(spec, inputs, got, tol, n=2000, kind="scale", seed=7):
    """Sampled comparison at n random cc points, each folded over its full pw range."""
    pts = oracle.random_points(spec, n, seed)
    lin, vals = oracle.evaluate_points(spec, inputs, pts)
    if kind == "scale":
        s2, ins2 = abs_spec_inputs(spec, inputs)
        _, svals = oracle.evaluate_points(s2, ins2, pts)
    for b, g in enumerate(got):
        gv = np.asarray(g).ravel()[lin[b]]
        o = vals[b]
        if spec["outputs"][b]["dtype"] not in FLOAT or kind == "exact":
            assert np.array_equal(gv.astype(o.dtype), o), f"output {b}: {np.count_nonzero(gv != o)} mismatches"
            continue
        g64 = gv.astype(np.float64) if spec["outputs"][b]["dtype"] != "bf16" else G.bf16_bits_to_f32(gv).astype(np.float64)
        err = np.abs(g64 - o)
        den = np.maximum(np.abs(o), 1e-300) if kind == "rel" else np.maximum(np.abs(svals[b]), 1e-300)
        assert (err / den).max() <= tol, f"max err {(err / den).max():.3e} > {tol}"
