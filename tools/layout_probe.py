"""Probe T4 throughput across operand layouts (K-major / MN-major A and B) and variants.

    python tools/layout_probe.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import bench
    from mdh_workloads import gen as G
    from mdh_workloads import specs as S
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device
    dev = torch.device("cuda", 0)
    flush = bench.L2Flush(dev)
    M = N = K = 4096
    d = ["i", "j", "k"]
    cases = []
    for at in (False, True):
        for bt in (False, True):
            a = ["k", "i"] if at else ["i", "k"]
            b = ["j", "k"] if bt else ["k", "j"]
            sp = S.make_spec("mm", d, [M, N, K], ["CC", "CC", "PW_ADD"], "MUL",
                             [S.buffer("A", "bf16", [a], d), S.buffer("B", "bf16", [b], d)],
                             [S.buffer("C", "f32", [["i", "j"]], d)])
            for tile in (None, "cluster=1"):
                cases.append((f"mm_{'T' if at else 'N'}{'T' if bt else 'N'}_{tile or 'auto'}", sp, tile, 2.0 * M * N * K))
    mcc = S.mcc(256, 7, 7, 512, 3, 3, 512, "bf16")
    for tile in (None, "implicit=1", "cluster=1"):
        cases.append((f"mcc_{tile or 'auto'}", mcc, tile, 2.0 * 256 * 49 * 512 * 4608))
    cases.append(("sgemm_f32", S.matmul(4096, 4096, 4096), None, 2.0 * 4096 ** 3))
    for name, sp, tile, flops in cases:
        plan = Plan(sp, force_tile=tile)
        host = G.gen_inputs(sp, 77) if not name.startswith("mcc") else G.mcc_inputs(sp)
        tin = [to_device(x, b["dtype"], dev) for x, b in zip(host, sp["inputs"])]
        outs = plan.empty_outputs(dev)
        ws = plan.workspace(dev) if plan.workspace_bytes else None
        step = lambda: plan(tin, outs, workspace_ptr=ws)
        for _ in range(3):
            step()
        torch.cuda.synchronize()
        ts = sorted(bench.time_steps(step, 10, torch.cuda.current_stream(), flush))
        med = ts[len(ts) // 2]
        print(json.dumps({"case": name, "us": round(med * 1e6, 1), "tflops": round(flops / med / 1e12, 1),
                          "variant": plan.describe().get("t4_variant"), "template": plan.template}), flush=True)
        del tin, outs, plan
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
