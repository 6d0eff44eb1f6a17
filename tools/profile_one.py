"""Run one bench workload a few times (for ncu captures; not a timing tool).

    python tools/profile_one.py --workload jacobi3d --reps 3
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", required=True)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--force-tile", default=None)
    a = ap.parse_args()
    import torch
    import bench
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device
    w = bench.workload(a.workload)
    dev = torch.device("cuda", 0)
    plan = Plan(w["spec"], force_tile=a.force_tile)
    tin = [to_device(x, b["dtype"], dev) for x, b in zip(w["inputs"](), w["spec"]["inputs"])]
    outs = plan.empty_outputs(dev)
    for _ in range(a.reps):
        plan(tin, outs)
    torch.cuda.synchronize()
    print(a.workload, plan.template, "launches/step", plan.last_launch_count())


if __name__ == "__main__":
    main()
