"""Quick device timing of bench workloads (median of CUDA-event pairs, L2 flushed).

    python tools/time_one.py ccsd_bf16 mcc_bf16 [--reps 10] [--force-tile split=4]
    ad-hoc shapes: mm:M,N,K (bf16 GEMM)  jac:Z,Y,X  prl:N,I  mcc:N,P,Q,K,R,S,C
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workloads", nargs="+")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--force-tile", default=None)
    a = ap.parse_args()
    import torch
    import bench
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device
    dev = torch.device("cuda", 0)
    pk = bench.peaks()
    flush = bench.L2Flush(dev)
    for name in a.workloads:
        if name.startswith("mm:"):          # ad-hoc bf16 GEMM shape "mm:M,N,K"
            from mdh_workloads import specs as S, gen as G
            M, N, K = (int(v) for v in name[3:].split(","))
            w = dict(spec=S.matmul(M, N, K, "bf16"), inputs=lambda M=M, N=N, K=K: G.matmul_inputs(M, N, K, "bf16"),
                     work=2.0 * M * N * K, unit="TFLOP/s", scale=1e12, bound="tensor", dtype="bf16")
        elif name.startswith("jac:"):         # Jacobi3D 7-pt over a Z×Y×X input (a z-slab with halos)
            from mdh_workloads import specs as S, gen as G
            Z, Y, X = (int(v) for v in name[4:].split(","))
            w = dict(spec=S.jacobi3d(Z, Y, X), inputs=lambda Z=Z, Y=Y, X=X: G.jacobi3d_inputs(Z, Y, X),
                     work=4.0 * (Z * Y * X + (Z - 2) * (Y - 2) * (X - 2)), unit="GB/s", scale=1e9, bound="hbm", dtype="f32")
        elif name.startswith("dot:"):         # fp32 Dot of N elements (read-only stream floor)
            from mdh_workloads import specs as S, gen as G
            N = int(name[4:])
            w = dict(spec=S.dot(N, "f32"), inputs=lambda N=N: G.dot_inputs(N, "f32"), work=8.0 * N,
                     unit="GB/s", scale=1e9, bound="hbm", dtype="f32")
        elif name.startswith("prl:"):         # PRL N new × I DB records
            from mdh_workloads import specs as S, gen as G
            N, I = (int(v) for v in name[4:].split(","))
            w = dict(spec=S.prl(N, I), inputs=lambda N=N, I=I: G.prl_inputs(N, I), work=float(N) * I,
                     unit="Gpairs/s", scale=1e9, bound="alu", dtype="u32")
        elif name.startswith("mcc:"):         # bf16 MCC N,P,Q,K,R,S,C
            from mdh_workloads import specs as S, gen as G
            cfg = [int(v) for v in name[4:].split(",")]
            sp = S.mcc(*cfg, dtype="bf16")
            w = dict(spec=sp, inputs=lambda sp=sp: G.mcc_inputs(sp), work=2.0 * cfg[0] * cfg[1] * cfg[2] * cfg[3] * cfg[4] * cfg[5] * cfg[6],
                     unit="TFLOP/s", scale=1e12, bound="tensor", dtype="bf16")
        else:
            w = bench.workload(name)
        plan = Plan(w["spec"], force_tile=a.force_tile)
        tin = [to_device(x, b["dtype"], dev) for x, b in zip(w["inputs"](), w["spec"]["inputs"])]
        outs = plan.empty_outputs(dev)
        if w.get("sweeps"):
            outs = [tin[0].clone()]
            step = lambda: plan.stencil_sweeps(tin[0], outs[0], w["sweeps"])
        else:
            step = lambda: plan(tin, outs)
        for _ in range(3):
            step()
        torch.cuda.synchronize()
        ts = sorted(bench.time_steps(step, a.reps, torch.cuda.current_stream(), flush))
        med = ts[len(ts) // 2]
        rl = bench.roofline(w, med, pk)
        print(json.dumps({"workload": name, "template": plan.template, "ms": round(med * 1e3, 4),
                          "value": round(w["work"] / med / w["scale"], 2), "unit": w["unit"],
                          "frac": round(rl["frac"], 4), "tiles": plan.describe()["tiles"]}), flush=True)
        del tin, outs, plan
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
