"""Quick device timing of bench workloads (median of CUDA-event pairs, L2 flushed).

    python tools/time_one.py ccsd_bf16 mcc_bf16 [--reps 10] [--force-tile split=4]
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
