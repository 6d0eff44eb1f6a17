"""Time arbitrary spec-builder expressions (CUDA events, L2 flushed), e.g.

    python tools/time_spec.py "S.ccsd_sd2()" "S.mcc(1, 7, 7, 512, 3, 3, 512, 'f32')" [--force-tile k=v]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("exprs", nargs="+")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--force-tile", default=None)
    a = ap.parse_args()
    import torch
    import bench
    from mdh_workloads import specs as S, gen as G   # noqa: F401 (used by the expressions)
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device
    dev = torch.device("cuda", 0)
    flush = bench.L2Flush(dev)
    for ex in a.exprs:
        spec = eval(ex)
        plan = Plan(spec, force_tile=a.force_tile)
        tin = [to_device(x, b["dtype"], dev) for x, b in zip(G.gen_inputs(spec, 9100), spec["inputs"])]
        outs = plan.empty_outputs(dev)
        for _ in range(3):
            plan(tin, outs)
        torch.cuda.synchronize()
        ts = sorted(bench.time_steps(lambda: plan(tin, outs), a.reps, torch.cuda.current_stream(), flush))
        print(json.dumps({"spec": ex, "template": plan.template, "ms": round(ts[len(ts) // 2] * 1e3, 4)}), flush=True)


if __name__ == "__main__":
    main()
