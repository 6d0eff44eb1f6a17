#!/usr/bin/env python
"""bench.py — throughput of the MDH hot path on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl mdh|reference]
                    [--workload NAME] [--no-suite]

A "step" is one mdh_execute of the whole hot path (plan not timed) on one batch of
synthetic input already resident in HBM.  The headline workload is BASELINE.json
configs[1]: MatMul 4096³, bf16 inputs / fp32 accumulate (`matmul_bf16`).  With N>1
(torchrun, one process per GPU) the SAME global problem is sharded (strong scaling,
SURVEY §8(e)): MatMul on M and Jacobi3D on z (cc shards, no communication), PRL A/B on
the DB dim and Dot 2^28 (pw shards: NCCL allgather + ordered combine inside
mdh_execute); T_p is the max over ranks and every rank's outputs are checked against
the oracle at sampled points.  MDH_BENCH_SAME_GPU=1 MDH_BENCH_BACKEND=gloo runs the N>1
harness with every rank on cuda:0 (VIRTUAL_SHARD plans; the pw partials are gathered
over torch.distributed and folded with mdh_combine_partials).

Timing: W untimed warm-up steps, then exactly K steps bracketed by barrier +
synchronize; each step's device time is a CUDA-event pair on the launching stream,
and the L2 is flushed (a 2×L2 memset, outside the event pair) before every step;
the reported time is the max over ranks.  Rank 0 prints ONE JSON line.  At N=1 the
line also carries `suite`: every §8 config measured the same way.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "per-workload GB/s or TFLOP/s and % of B200 roofline, at 1/2/4/8 GPUs"
FALLBACK = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}
# derived unit-count peaks, used only when the on-box measurement
# (mdh_measure_peaks) is unavailable
FFMA_TFLOPS = 148 * 128 * 2 * 1.965e9 / 1e12     # fp32 FFMA
ALU_TOPS = 148 * 4 * 32 * 1.965e9 / 1e12         # thread-instructions/s issue


_PIPE = {}


def pipe_peaks(device=0):
    """FFMA / issue peaks measured on this GPU (mdh_measure_peaks, once per process)."""
    if "v" not in _PIPE:
        try:
            from paper_conf_sc_schulzegr25_b200 import measure_peaks
            m = measure_peaks(device)
            _PIPE["v"] = {"ffma_tflops": m["ffma_tflops"], "issue_tops": m["issue_tops"], "alu_tops": m["alu_tops"],
                          "source": "measured on this GPU (mdh_measure_peaks: FFMA chains; issue = best sustained instruction rate)"}
        except Exception as e:  # no GPU / measurement failed: derived unit-count peaks
            _PIPE["v"] = {"ffma_tflops": FFMA_TFLOPS, "issue_tops": ALU_TOPS, "alu_tops": ALU_TOPS / 2,
                          "source": f"derived from unit counts and 1.965 GHz ({str(e)[:60]})"}
    return _PIPE["v"]


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return {"hbm_gbs": d.get("hbm_gbs", FALLBACK["hbm_gbs"]), "bf16_tflops": d.get("bf16_tflops", FALLBACK["bf16_tflops"]),
                "bf16_tflops_sustained": d.get("bf16_tflops_sustained", FALLBACK["bf16_tflops_sustained"]),
                "source": "measured (MEASURED_PEAKS.json)"}
    return dict(FALLBACK, source="fallback (B200_PROFILING.md)")


# ------------------------------------------------------------------------------ workloads
def workload(name):
    """The GLOBAL configuration of a workload: spec, seeded host-input generator, algorithmic
    work of the whole problem, unit, roofline kind and — for the configs SURVEY §8(e)
    shards — the shard dim (a cc dim: no communication; a pw dim: allgather + ordered
    combine over NCCL).  With N GPUs every rank plans its sub-domain of this global problem
    (strong scaling) and slices its inputs with mdh_plan_local_shape."""
    from mdh_workloads import gen as G
    from mdh_workloads import specs as S
    if name in ("matmul_bf16", "matmul_f32"):
        dt = "bf16" if name == "matmul_bf16" else "f32"
        spec = S.matmul(4096, 4096, 4096, dt)
        return dict(spec=spec, inputs=lambda: list(G.matmul_inputs(4096, 4096, 4096, dt, "signed", seed_base=2000)),
                    work=2.0 * 4096 ** 3, unit="TFLOP/s", scale=1e12,
                    bound="tensor" if dt == "bf16" else "alu", shard_dim=0, dtype=dt,
                    desc=f"MatMul 4096x4096x4096 {dt} (Listing 9), {'tcgen05' if dt == 'bf16' else 'FFMA'} path")
    if name.startswith("dot"):
        dt = "i32" if "i32" in name else "f32"
        N = 1 << 28 if name.endswith("2^28") else 1 << 20
        spec = S.dot(N, dt)
        return dict(spec=spec, inputs=lambda: G.dot_inputs(N, dt, "signed"), work=8.0 * N + 4, unit="GB/s",
                    scale=1e9, bound="hbm", dtype=dt, shard_dim=0, desc=f"Dot N={N} {dt} (Fig 3 P:512)")
    if name == "matvec_f32":
        spec = S.matvec(8192, 8192)
        return dict(spec=spec, inputs=lambda: G.gen_inputs(spec, 2100), work=4.0 * (8192 * 8192 + 8192 + 8192),
                    unit="GB/s", scale=1e9, bound="hbm", dtype="f32", desc="MatVec 8192^2 fp32 (Listing 6)")
    if name == "jacobi3d":
        spec = S.jacobi3d(512, 512, 512)
        return dict(spec=spec, inputs=lambda: G.jacobi3d_inputs(512, 512, 512), work=4.0 * (512 ** 3 + 510 ** 3),
                    unit="GB/s", scale=1e9, bound="hbm", dtype="f32", shard_dim=0, desc="Jacobi3D 7-pt 512^3 fp32")
    if name == "jacobi3d_sweeps8":
        T = 8
        spec = S.jacobi3d_sweep(512, 512, 512)
        return dict(spec=spec, inputs=lambda: G.jacobi3d_inputs(512, 512, 512), work=T * 4.0 * (512 ** 3 + 510 ** 3),
                    unit="GB/s", scale=1e9, bound="hbm", dtype="f32", sweeps=T,
                    desc="Jacobi3D 7-pt 512^3 fp32, 8 sweeps u->v->u (mdh_stencil_sweeps; F3, reading C-34)")
    if name == "ccsd_bf16":
        spec = S.ccsd_sd1(24, 72, "bf16")
        out = 24 ** 3 * 72 ** 3
        return dict(spec=spec, inputs=lambda: G.gen_inputs(spec, 4000), work=4.0 * out + 2.0 * (72 ** 2 * 24 ** 2 + 72 ** 3 * 24),
                    unit="GB/s", scale=1e9, bound="hbm", dtype="bf16", flops=2.0 * out * 72,
                    desc="CCSD(T) sd1 O=24 V=72 bf16->fp32 (HBM-bound on the 20.6 GB output)")
    if name == "mcc_bf16":
        spec = S.mcc(256, 7, 7, 512, 3, 3, 512, "bf16")
        return dict(spec=spec, inputs=lambda: G.mcc_inputs(spec), work=2.0 * 256 * 49 * 512 * 4608, unit="TFLOP/s",
                    scale=1e12, bound="tensor", dtype="bf16", desc="MCC ResNet-50 conv5_1 3x3/s2 N=256 bf16")
    if name == "mcc_conv1_bf16":
        # C4b-B (reading C-21): conv1 7x7/s2, C=3, K=64, P=Q=112 at N=256 — HBM-bound on its
        # 822 MB fp32 output (bytes: image + filter read once, output written once)
        spec = S.mcc(256, 112, 112, 64, 7, 7, 3, "bf16")
        byts = 2.0 * 256 * 230 * 230 * 3 + 2.0 * 64 * 147 + 4.0 * 256 * 112 * 112 * 64
        return dict(spec=spec, inputs=lambda: G.mcc_inputs(spec), work=byts, unit="GB/s", scale=1e9, bound="hbm",
                    dtype="bf16", flops=2.0 * 256 * 112 * 112 * 64 * 147,
                    desc="MCC ResNet-50 conv1 7x7/s2 N=256 bf16->fp32 (Fig 3 MCC Inp.2; HBM-bound on the 822 MB output)")
    if name == "mcc_bf16_n1":
        spec = S.mcc(1, 7, 7, 512, 3, 3, 512, "bf16")
        return dict(spec=spec, inputs=lambda: G.mcc_inputs(spec), work=2.0 * 49 * 512 * 4608, unit="TFLOP/s",
                    scale=1e12, bound="tensor", dtype="bf16", desc="MCC ResNet-50 conv5_1 3x3/s2 N=1 bf16 (the paper's batch)")
    if name == "gaussian2d":
        I = J = 4096
        spec = S.gaussian2d(I, J)
        return dict(spec=spec, inputs=lambda: G.gaussian2d_inputs(I, J), work=4.0 * ((I + 4) * (J + 4) + I * J),
                    unit="GB/s", scale=1e9, bound="hbm", dtype="f32",
                    desc="Gaussian_2D 5x5 4096^2 fp32 (Fig 3 P:520-521; reading C-31)")
    if name == "matvec_4096":
        spec = S.matvec(4096, 4096)
        return dict(spec=spec, inputs=lambda: G.gen_inputs(spec, 2100), work=4.0 * (4096 * 4096 + 4096 + 4096),
                    unit="GB/s", scale=1e9, bound="hbm", dtype="f32", desc="MatVec 4096^2 fp32 (Fig 3 P:514)")
    if name == "mcc_caps_bf16":
        spec = S.mcc_caps(16, 112, 112, 64, 7, 7, 3, dtype="bf16")
        return dict(spec=spec, inputs=lambda: G.gen_inputs(spec, 4300), work=2.0 * 16 * 112 * 112 * 64 * 16 * 588,
                    unit="TFLOP/s", scale=1e12, bound="tensor", dtype="bf16",
                    desc="MCC_Caps 16x230x230x3x4x4 * 64x7x7x3x4x4 bf16 (Fig 3 P:530; reading C-33)")
    if name == "prefix_sum_f32":
        spec = S.prefix_sum([1 << 26], 0)
        return dict(spec=spec, inputs=lambda: G.gen_inputs(spec, 6100, "positive"), work=8.0 * (1 << 26),
                    unit="GB/s", scale=1e9, bound="hbm", dtype="f32",
                    desc="ps(add) prefix sum of 2^26 fp32 (Listing 17; F1)")
    if name == "mbbs_f32":
        spec = S.mbbs(8192, 8192)
        return dict(spec=spec, inputs=lambda: G.gen_inputs(spec, 6200, "positive"), work=4.0 * (8192 * 8192 + 8192),
                    unit="GB/s", scale=1e9, bound="hbm", dtype="f32",
                    desc="MBBS md_hom(id,(pw(add),ps(add))) over 8192^2 fp32 (F1)")
    if name in ("prl_A", "prl_B"):
        N, I = ((1 << 20), (1 << 14)) if name == "prl_A" else ((1 << 14), (1 << 20))
        spec = S.prl(N, I)
        return dict(spec=spec, inputs=lambda: G.prl_inputs(N, I), work=float(N) * I, unit="Gpairs/s", scale=1e9,
                    bound="alu", dtype="u32", shard_dim=1, desc=f"PRL {N}x{I} custom argmax (Listing 11)")
    raise SystemExit(f"unknown workload {name}")


# configs sharded at N > 1: the headline plus these, each strong-scaled
SHARDED = ["jacobi3d", "prl_A", "prl_B", "dot_f32_2^28"]
SUITE = ["dot_f32", "dot_i32", "dot_f32_2^28", "matvec_f32", "matvec_4096", "jacobi3d", "jacobi3d_sweeps8", "gaussian2d", "matmul_f32",
         "matmul_bf16", "ccsd_bf16", "mcc_bf16", "mcc_conv1_bf16", "mcc_bf16_n1", "mcc_caps_bf16", "prl_A", "prl_B", "prefix_sum_f32", "mbbs_f32"]


def roofline(w, seconds, pk):
    """achieved algorithmic rate of the dominant kernel vs the measured peak."""
    if w["bound"] == "hbm":
        ach = w["work"] / seconds / 1e9
        return {"bound": "hbm", "achieved": ach, "peak": pk["hbm_gbs"], "unit": "GB/s", "frac": ach / pk["hbm_gbs"]}
    if w["bound"] == "tensor":
        ach = w["work"] / seconds / 1e12
        peak = pk["bf16_tflops"]
        return {"bound": "tensor", "achieved": ach, "peak": peak, "unit": "TFLOP/s", "frac": ach / peak}
    pp = pipe_peaks()
    if w["unit"] == "TFLOP/s":     # fp32 SIMT: the FFMA pipe, measured on the box
        ach = w["work"] / seconds / 1e12
        return {"bound": "alu", "achieved": ach, "peak": pp["ffma_tflops"], "unit": "TFLOP/s",
                "frac": ach / pp["ffma_tflops"], "peak_source": pp["source"]}
    # PRL: 9 algorithmic ops per pair (8 field compares + 1 combine) against the
    # measured instruction-issue rate (the kernel feeds both the ALU and the FMA pipe)
    ach = w["work"] * 9 / seconds / 1e12
    return {"bound": "alu", "achieved": ach, "peak": pp["issue_tops"], "unit": "Tops/s",
            "frac": ach / pp["issue_tops"], "peak_source": pp["source"]}


class Clocks:
    """nvidia-smi sampler run DURING the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index):
        self.index = index
        self.p = None

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={q}", "--format=csv,noheader,nounits", "-lms", "50",
                                       "-i", str(self.index)], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.p = None
        time.sleep(0.15)
        return self

    def __exit__(self, *a):
        self.summary = None
        if not self.p:
            return
        time.sleep(0.1)
        self.p.terminate()
        out, _ = self.p.communicate(timeout=10)
        rows = [r.split(", ") for r in out.strip().splitlines() if r.count(",") >= 5]
        if not rows:
            return
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in rows for k in range(4) if r[2 + k].strip() == "Active"})
        self.summary = {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                        "reasons": reasons, "samples": len(rows)}


class L2Flush:
    """Evicts the L2 before a timed step: write a 2×L2 buffer, then read another 2×L2
    buffer, so the step starts with an L2 holding clean, unrelated lines (no write-back
    of flush data is charged to the timed step)."""

    def __init__(self, dev):
        import torch
        n = 2 * torch.cuda.get_device_properties(dev).L2_cache_size // 4
        self.w = torch.empty(n, dtype=torch.float32, device=dev)
        self.r = torch.ones(n, dtype=torch.float32, device=dev)
        self.sink = torch.empty((), dtype=torch.float32, device=dev)

    def zero_(self):
        import torch
        self.w.zero_()
        torch.sum(self.r, dim=0, out=self.sink)


def time_steps(step, K, stream, flush):
    import torch
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    for k in range(K):
        if flush is not None:
            flush.zero_()
        ev[k][0].record(stream)
        step()
        ev[k][1].record(stream)
    torch.cuda.synchronize()
    return [a.elapsed_time(b) / 1e3 for a, b in ev]


def hot_time(step, dev, n=20, reps=5):
    """Hot-L2 time per execute: n back-to-back executes captured in one CUDA
    graph, replayed `reps` times, total ÷ (n·reps).  Not compared to the HBM roofline (the
    operands stay in L2); None when the path cannot be captured."""
    import torch
    try:
        s = torch.cuda.Stream(dev)
        with torch.cuda.stream(s):
            step(s.cuda_stream)
        s.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(n):
                step(s.cuda_stream)
        g.replay()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            g.replay()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / 1e3 / (n * reps)
    except Exception:  # capture unsupported on this path: report no hot number
        torch.cuda.synchronize()
        return None


def run_mdh_workload(name, K, W, world, rank, dev, flush, pk, with_e2e=False, check=False, ci=False):
    import torch
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device
    w = workload(name)
    plan = Plan(w["spec"], device=dev)
    host = w["inputs"]()
    tin = [to_device(x, b["dtype"], dev) for x, b in zip(host, w["spec"]["inputs"])]
    outs = plan.empty_outputs(dev)
    ws = plan.workspace(dev) if plan.workspace_bytes else None
    stream = torch.cuda.current_stream(dev)
    sh = stream.cuda_stream

    if w.get("sweeps"):                     # time-stepping: the output buffer is the second field
        outs = [tin[0].clone()]

        def step(h=sh):
            plan.stencil_sweeps(tin[0], outs[0], w["sweeps"], stream=h, workspace_ptr=ws)
    else:
        def step(h=sh):
            plan(tin, outs, stream=h, workspace_ptr=ws)
    # warm-up steps are the timed steps' exact sequence (L2 flush, then the step), so the first
    # timed step is not the first one after a flush (it measured 178 µs vs ~103 µs otherwise)
    for _ in range(W):
        if flush is not None:
            flush.zero_()
        step()
    torch.cuda.synchronize()
    launches = plan.last_launch_count()
    # the headline times exactly K steps (driver contract); suite entries follow the
    # paper's stopping rule (99 % CI half-width within 5 %, capped)
    times = time_until_ci(step, K, stream, flush) if ci else time_steps(step, K, stream, flush)
    res = {"plan": plan, "w": w, "times": times, "launches": launches, "host": host, "outs": outs}
    res["hot"] = hot_time(step, dev)
    if with_e2e:
        # end to end through mdh_execute_host: pinned host in/out, copies inside the events
        hin = [torch.from_numpy(np.ascontiguousarray(x).view(np.int16) if b["dtype"] == "bf16" else np.ascontiguousarray(x)).pin_memory()
               for x, b in zip(host, w["spec"]["inputs"])]
        hout = [torch.empty(o.shape, dtype=o.dtype).pin_memory() for o in outs]
        nscr = plan.host_scratch_bytes()
        scratch = torch.empty(nscr, dtype=torch.uint8, device=dev)

        def e2e_step():
            plan.execute_host(hin, hout, scratch.data_ptr(), nscr, sh)
        for _ in range(W):
            e2e_step()
        torch.cuda.synchronize()
        et = time_steps(e2e_step, K, stream, None)
        res["e2e_times"] = et
        res["h2d"] = int(sum(t.numel() * t.element_size() for t in hin))
        res["d2h"] = int(sum(t.numel() * t.element_size() for t in hout))
    if check:
        import oracle
        from paper_conf_sc_schulzegr25_b200 import to_numpy
        pts = oracle.random_points(w["spec"], 256, seed=11)
        lin, vals = oracle.evaluate_points(w["spec"], host, pts)
        g = to_numpy(outs[0], w["spec"]["outputs"][0]["dtype"]).ravel()[lin[0]].astype(np.float64)
        ref = vals[0]
        res["parity"] = {"points": 256, "max_rel_err": float(np.max(np.abs(g - ref) / np.maximum(np.abs(ref), 1e-30)))}
    return res


def ci99_halfwidth(times):
    """Student-t 99 % confidence half-width of the mean of `times`, as a fraction of the mean
    (the paper's stopping rule)."""
    n = len(times)
    if n < 2:
        return None
    m = float(np.mean(times))
    sd = float(np.std(times, ddof=1))
    try:
        from scipy.stats import t as student_t
        q = float(student_t.ppf(0.995, n - 1))
    except Exception:  # scipy missing: normal quantile (slightly optimistic for small n)
        q = 2.576
    return q * sd / np.sqrt(n) / m if m > 0 else None


def time_until_ci(step, K, stream, flush, rel=0.05, cap_reps=200, cap_s=10.0):
    """At least K repetitions, then more until the 99 % CI half-width is within `rel` of
    the mean, capped at cap_reps repetitions or cap_s seconds of device time."""
    times = time_steps(step, K, stream, flush)
    while len(times) < cap_reps and sum(times) < cap_s:
        h = ci99_halfwidth(times)
        if h is not None and h <= rel:
            break
        times += time_steps(step, max(K, len(times) // 2), stream, flush)
    return times


# ------------------------------------------------------------------------- N > 1 (§8(e))
def log(*a):
    """Progress to stderr (MDH_BENCH_VERBOSE=1)."""
    if os.environ.get("MDH_BENCH_VERBOSE") == "1":
        print(f"[rank {os.environ.get('RANK', '0')} {time.strftime('%H:%M:%S')}]", *a, file=sys.stderr, flush=True)


def slice_local(x, shape, off):
    return np.ascontiguousarray(x[tuple(slice(o, o + n) for o, n in zip(off, shape))])


def run_sharded(name, K, W, world, rank, dev, flush, comm, virtual, with_e2e=False, npts=256):
    """One strong-scaled sharded workload on this rank: plan the rank's sub-domain of the
    global problem (mdh_plan with world_size/rank/shard_dim), slice the seeded global
    inputs with mdh_plan_local_shape, time K executes (barrier + synchronize before each,
    L2 flushed outside the event pair; a pw shard's execute includes the NCCL allgather
    and the ordered combine), then check sampled outputs against the oracle.  With
    `virtual` (one GPU shared by every rank: MDH_BENCH_SAME_GPU=1) the plans are
    VIRTUAL_SHARD — no NCCL; a pw shard's partials are gathered over torch.distributed
    and folded on rank 0 with mdh_combine_partials, standing in for the allgather."""
    import torch
    import torch.distributed as dist
    import oracle
    from paper_conf_sc_schulzegr25_b200 import VIRTUAL_SHARD, Plan, to_device, to_numpy
    w = workload(name)
    spec = w["spec"]
    sd = w["shard_dim"]
    kw = dict(world_size=world, rank=rank, shard_dim=sd)
    if virtual:
        kw["flags"] = VIRTUAL_SHARD
    else:
        kw["comm"] = comm
    log(name, "plan")
    plan = Plan(spec, device=dev, **kw)
    desc = plan.describe()
    host = w["inputs"]()
    local = [slice_local(x, *plan.local_shape(False, b)[:2]) for b, x in enumerate(host)]
    log(name, "inputs sliced", [x.shape for x in local])
    tin = [to_device(x, bb["dtype"], dev) for x, bb in zip(local, spec["inputs"])]
    outs = plan.empty_outputs(dev)
    ws = plan.workspace(dev) if plan.workspace_bytes else None
    stream = torch.cuda.current_stream(dev)
    sh = stream.cuda_stream

    def step():
        plan(tin, outs, stream=sh, workspace_ptr=ws)
    for _ in range(W):
        step()
    torch.cuda.synchronize()
    log(name, "warm")
    launches = plan.last_launch_count()
    times = []
    for _ in range(K):
        flush.zero_()
        torch.cuda.synchronize()
        dist.barrier()
        times += time_steps(step, 1, stream, None)
    res = {"plan": plan, "w": w, "desc": desc, "times": times, "launches": launches}
    if with_e2e:
        hin = [torch.from_numpy(np.ascontiguousarray(x).view(np.int16) if bb["dtype"] == "bf16" else np.ascontiguousarray(x)).pin_memory()
               for x, bb in zip(local, spec["inputs"])]
        hout = [torch.empty(o.shape, dtype=o.dtype).pin_memory() for o in outs]
        nscr = plan.host_scratch_bytes()
        scratch = torch.empty(nscr, dtype=torch.uint8, device=dev)
        et = []
        for k in range(W + K):
            torch.cuda.synchronize()
            dist.barrier()
            t = time_steps(lambda: plan.execute_host(hin, hout, scratch.data_ptr(), nscr, sh), 1, stream, None)
            if k >= W:
                et += t
        res["e2e_times"] = et
        res["h2d"] = int(sum(t.numel() * t.element_size() for t in hin))
        res["d2h"] = int(sum(t.numel() * t.element_size() for t in hout))
    log(name, "timed", times)
    # ---- parity: sampled global points against the oracle
    pw = spec["ops"][sd] != "CC"
    nin = len(spec["inputs"])
    gshapes = oracle.shapes(spec)[nin:]
    got = [to_numpy(o, b["dtype"]) for o, b in zip(outs, spec["outputs"])]
    if pw and virtual:
        allp = [None] * world
        dist.all_gather_object(allp, got)
        if rank == 0:
            parts = [[to_device(a, b["dtype"], dev) for a, b in zip(pr, spec["outputs"])] for pr in allp]
            fin = plan.combine_partials(parts)
            torch.cuda.synchronize()
            got = [to_numpy(o, b["dtype"]) for o, b in zip(fin, spec["outputs"])]
    if all(o != "CC" for o in spec["ops"]):
        npts = 1                    # no cc dim (Dot): one output, one full fold
    pts = oracle.random_points(spec, npts, seed=11 + rank)
    if not pw:
        lo, n = desc["shard_start"], desc["shard_len"]
        pts = pts[(pts[:, sd] >= lo) & (pts[:, sd] < lo + n)]
    ok, err = True, 0.0
    if len(pts) and (not (pw and virtual) or rank == 0):
        lin, vals = oracle.evaluate_points(spec, host, pts)
        for b, (g, o) in enumerate(zip(got, vals)):
            shp, off, _ = plan.local_shape(True, b)
            idx = np.unravel_index(lin[b], gshapes[b])
            loc = np.ravel_multi_index(tuple(i - f for i, f in zip(idx, off)), shp)
            gv = np.asarray(g).ravel()[loc]
            dt = spec["outputs"][b]["dtype"]
            if dt in ("f32", "f64", "bf16"):
                e = float(np.max(np.abs(gv.astype(np.float64) - o)) / max(float(np.max(np.abs(o))), 1e-30))
                err = max(err, e)
                ok &= e <= (1e-2 if w["dtype"] == "bf16" else 1e-4)
            else:
                ok &= bool(np.array_equal(gv.astype(o.dtype), o))
    log(name, "parity", ok, err)
    res["parity"] = {"points": int(len(pts)), "ok": bool(ok), "max_normwise_err": err,
                     "how": "sampled global points vs the fp64 oracle; exact for integer/PRL outputs"}
    return res


def sharded_main(a, W, K, world, rank, local, dev, backend):
    """N > 1: strong scaling of the global problems of SURVEY §8(e) — MatMul 4096³ on M,
    Jacobi3D 512³ on z (cc shards, no communication), PRL A/B on the DB dim and Dot 2^28
    (pw shards: NCCL allgather + ordered combine) — T_p = max over ranks."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_schulzegr25_b200 import Comm
    virtual = os.environ.get("MDH_BENCH_SAME_GPU") == "1"
    log("sharded main, virtual =", virtual)
    comm = None if virtual else Comm(device=dev)
    pk = peaks()
    flush = L2Flush(dev)
    red_dev = dev if backend == "nccl" else "cpu"

    def tmax(vals):
        t = torch.tensor(vals, dtype=torch.float64, device=red_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return [float(v) for v in t.cpu()]

    def gather(obj):
        out = [None] * world
        dist.all_gather_object(out, obj)
        return out

    def entry(r, with_line=False):
        w = r["w"]
        tt = tmax([sum(r["times"])] + ([sum(r["e2e_times"])] if "e2e_times" in r else []))
        per = tt[0] / len(r["times"])
        par = gather(r["parity"])
        kind = "cc" if w["spec"]["ops"][w["shard_dim"]] == "CC" else "pw"
        e = {"value": round(w["work"] / per / w["scale"], 3), "unit": w["unit"], "ms_per_step": round(per * 1e3, 4),
             "template": r["plan"].template, "launches_per_step": r["launches"], "roofline_1gpu_equiv":
             roofline(w, per * world, pk), "ci99_halfwidth_pct": round(100 * (ci99_halfwidth(r["times"]) or 0), 2),
             "shard": {"dim": w["shard_dim"], "kind": kind,
                       "exchange": "none (cc shard)" if kind == "cc" else
                       ("allgather over torch.distributed + mdh_combine_partials (virtual, one GPU)" if virtual
                        else "NCCL allgather + ordered combine inside mdh_execute")},
             "parity": {"ok": all(p["ok"] for p in par), "points": sum(p["points"] for p in par),
                        "max_normwise_err": max(p["max_normwise_err"] for p in par)},
             "desc": w["desc"]}
        if "e2e_times" in r:
            e["e2e_value"] = round(w["work"] / (tt[1] / len(r["e2e_times"])) / w["scale"], 3)
        return e, per, tt

    dist.barrier()
    torch.cuda.synchronize()
    with Clocks(local) as clk:
        res = run_sharded(a.workload, K, W, world, rank, dev, flush, comm, virtual, with_e2e=True)
        dist.barrier()
        torch.cuda.synchronize()
    head, per, tt = entry(res)
    w = res["w"]
    line = {"metric": METRIC, "value": head["value"], "unit": w["unit"], "n_gpus": world, "steps": K, "warmup": W,
            "ms_per_step": head["ms_per_step"], "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": w["dtype"], "data": "synthetic (seeded numpy PCG64, shapes of Fig 3 / SURVEY §8(d))",
            "config": {"workload": a.workload, "desc": w["desc"], "template": res["plan"].template,
                       "global_shape": w["spec"]["sizes"],
                       "l2": "flushed before every step (2xL2 write, then 2xL2 read of another buffer), outside the event pair",
                       "parallelism": f"{head['shard']['kind']} shard of dim {w['shard_dim']} over {world} GPUs "
                                      f"({head['shard']['exchange']})", "virtual_ranks_on_one_gpu": virtual},
            "roofline": dict(head["roofline_1gpu_equiv"], note="achieved per GPU-equivalent: work / (T_p x N)",
                             peak_source=pk["source"]),
            "e2e": {"value": head.get("e2e_value"), "unit": w["unit"], "h2d_bytes_per_step": res["h2d"],
                    "d2h_bytes_per_step": res["d2h"], "api": "mdh_execute_host per rank (pinned host slices)"},
            "gpu_launches": res["launches"] * K, "ci99_halfwidth_pct": head["ci99_halfwidth_pct"],
            "parity_sample": head["parity"], "clocks": clk.summary}
    del res
    if not a.no_suite:
        suite = {}
        for name in SHARDED:
            if name == a.workload:
                continue
            try:
                r = run_sharded(name, a.suite_steps, 3, world, rank, dev, flush, comm, virtual,
                                npts=64 if name == "prl_B" else 256)
                suite[name] = entry(r)[0]
                del r
            except Exception as e:  # keep the headline even if a suite member fails
                suite[name] = {"error": str(e)[:300]}
            torch.cuda.empty_cache()
        line["suite"] = suite
    if rank == 0:
        print(json.dumps(line), flush=True)
    dist.barrier()
    if comm is not None:
        comm.close()
    dist.destroy_process_group()
    return 0


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for l in f:
                if l.startswith("model name"):
                    return l.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_baseline(w, target_s=12.0):
    """The oracle as it stands, on this host's cores, on a bounded sample of the workload."""
    import oracle
    spec = w["spec"]
    host = w["inputs"]()
    n = 16
    t = 0.0
    while True:
        pts = oracle.random_points(spec, n, seed=3)
        t0 = time.perf_counter()
        oracle.evaluate_points(spec, host, pts)
        t = time.perf_counter() - t0
        if t > target_s / 4 or n >= 1 << 22:
            break
        n *= 4 if t < target_s / 64 else 2
    ncc = 1
    for s, o in zip(spec["sizes"], spec["ops"]):
        if o == "CC":
            ncc *= s
    frac = n / ncc
    value = w["work"] * frac / t / w["scale"]
    return {"value": value, "unit": w["unit"], "cores": oracle.max_threads(), "cpu_model": cpu_model(), "kind": "oracle",
            "sample": f"{n} random output points of {w['desc']} ({frac:.2e} of the work), each folded over its full "
                      f"reduction range by the literal fp64 loop nest; {t:.1f} s"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="mdh", choices=["mdh", "reference"])
    ap.add_argument("--workload", default="matmul_bf16")
    ap.add_argument("--no-suite", action="store_true")
    ap.add_argument("--suite-steps", type=int, default=10)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    a = ap.parse_args()
    W = max(3, a.warmup)
    K = max(1, a.steps)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))

    if a.impl == "reference":
        return reference_arm(a, W, K, world, rank)

    import torch
    import torch.distributed as dist
    from paper_conf_sc_schulzegr25_b200 import lib
    lib()
    # MDH_BENCH_BACKEND=gloo and MDH_BENCH_SAME_GPU=1 exercise the N>1 launch on a
    # single-GPU machine (every rank on cuda:0); the default is NCCL, one GPU per rank.
    backend = os.environ.get("MDH_BENCH_BACKEND", "nccl")
    local = 0 if os.environ.get("MDH_BENCH_SAME_GPU") == "1" else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    if world > 1:
        return sharded_main(a, W, K, world, rank, local, dev, backend)
    pk = peaks()
    flush = L2Flush(dev)

    # ---- headline (one GPU: barrier = device synchronize)
    torch.cuda.synchronize()
    with Clocks(local) as clk:
        torch.cuda.synchronize()
        res = run_mdh_workload(a.workload, K, W, world, rank, dev, flush, pk, with_e2e=True, check=True)
        torch.cuda.synchronize()
    t_total = sum(res["times"])
    et_total = sum(res["e2e_times"])
    w = res["w"]
    per_step = t_total / K
    value = w["work"] / per_step / w["scale"]
    e2e_value = w["work"] / (et_total / K) / w["scale"]
    rl = roofline(w, per_step, pk)
    rl["peak_source"] = pk["source"]
    rl["traffic"] = ncu_traffic(a.workload)
    rl["kernel"] = res["plan"].template
    line = {"metric": METRIC, "value": round(value, 3), "unit": w["unit"], "n_gpus": world, "steps": K, "warmup": W,
            "ms_per_step": round(per_step * 1e3, 4), "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": w["dtype"], "data": "synthetic (seeded numpy PCG64, shapes of Fig 3 / SURVEY §8(d))",
            "config": {"workload": a.workload, "desc": w["desc"], "template": res["plan"].template,
                       "global_shape": w["spec"]["sizes"], "l2": "flushed before every step (2xL2 write, then 2xL2 read of another buffer), outside the event pair",
                       "parallelism": "1 GPU (N > 1: the same global problem sharded, SURVEY §8(e))"},
            "ci99_halfwidth_pct": round(100 * (ci99_halfwidth(res["times"]) or 0), 2),
            "roofline": rl,
            "e2e": {"value": round(e2e_value, 3), "unit": w["unit"], "h2d_bytes_per_step": res["h2d"],
                    "d2h_bytes_per_step": res["d2h"], "api": "mdh_execute_host (pinned host buffers)"},
            "gpu_launches": res["launches"] * K,
            "hot": ({"ms_per_execute": round(res["hot"] * 1e3, 4), "value": round(w["work"] / res["hot"] / w["scale"], 3),
                     "how": "20 executes captured in one CUDA graph, L2 warm (not a roofline number)"}
                    if res.get("hot") else None),
            "clocks": clk.summary}
    if "parity" in res:
        line["parity_sample"] = res["parity"]
    del res
    # ---- suite of every §8 config (N=1)
    if not a.no_suite:
        suite = {}
        for name in SUITE:
            if name == a.workload:
                continue
            try:
                r = run_mdh_workload(name, a.suite_steps, 3, 1, 0, dev, flush, pk, ci=True)
                ts = sorted(r["times"])
                med = ts[len(ts) // 2]
                ww = r["w"]
                ent = {"value": round(ww["work"] / med / ww["scale"], 3), "unit": ww["unit"], "ms_median": round(med * 1e3, 4),
                       "reps": len(ts), "ci99_halfwidth_pct": round(100 * (ci99_halfwidth(ts) or 0), 2),
                       "hot_ms": round(r["hot"] * 1e3, 4) if r.get("hot") else None,
                       "template": r["plan"].template, "launches_per_step": r["launches"],
                       "roofline": roofline(ww, med, pk), "desc": ww["desc"]}
                if "flops" in ww:
                    ent["tflops"] = round(ww["flops"] / med / 1e12, 2)
                suite[name] = ent
                del r
            except Exception as e:  # keep the headline even if a suite member fails
                suite[name] = {"error": str(e)[:300]}
            torch.cuda.empty_cache()
        line["suite"] = suite
    if not a.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(workload(a.workload))
    print(json.dumps(line), flush=True)


def ncu_traffic(name):
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f).get(name)
    return None


def reference_arm(a, W, K, world, rank):
    """--impl reference: the oracle (CPU loop nest) as it stands, on this host's cores,
    each step a bounded sample of the same workload; rank 0 only."""
    if rank != 0:
        return 0
    import oracle
    w = workload(a.workload)
    spec, host = w["spec"], w["inputs"]()
    n = 64
    while True:     # size one step to ~4 s so that W+K steps end within a few minutes
        pts = oracle.random_points(spec, n, seed=5)
        t0 = time.perf_counter()
        oracle.evaluate_points(spec, host, pts)
        t = time.perf_counter() - t0
        if t > 1.0 or n >= 1 << 22:
            break
        n *= 2
    budget = 150.0
    n = max(16, int(n * min(4.0, budget / (W + K)) / max(t, 1e-3)))
    times = []
    for k in range(W + K):
        pts = oracle.random_points(spec, n, seed=100 + k)
        t0 = time.perf_counter()
        oracle.evaluate_points(spec, host, pts)
        if k >= W:
            times.append(time.perf_counter() - t0)
    ncc = 1
    for s, o in zip(spec["sizes"], spec["ops"]):
        if o == "CC":
            ncc *= s
    frac = n / ncc
    per = sum(times) / len(times)
    value = w["work"] * frac / per / w["scale"]
    line = {"metric": METRIC, "value": value, "unit": w["unit"], "n_gpus": world, "steps": K, "warmup": W,
            "ms_per_step": per * 1e3, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": w["dtype"], "data": "synthetic", "impl": "reference",
            "config": {"workload": a.workload, "desc": w["desc"]},
            "cpu_baseline": {"value": value, "unit": w["unit"], "cores": oracle.max_threads(), "cpu_model": cpu_model(), "kind": "oracle",
                             "sample": f"{n} random output points per step ({frac:.2e} of the work), literal fp64 loop nest"},
            "e2e": {"value": value, "unit": w["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


if __name__ == "__main__":
    sys.exit(main())
