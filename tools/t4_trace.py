"""Diagnostics: per-unit timeline of the T4 2-SM kernel (MDH_T4_TRACE=1).

    MDH_T4_TRACE=1 python tools/t4_trace.py mcc_bf16 mm:12544,512,4608 [--force-tile split=2]

Prints, per workload: kernel span, unit durations (first MMA → last commit) by wave, and
the per-pair busy time, so wave quantisation and per-k-block rates can be read directly.
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
    ap.add_argument("--force-tile", default=None)
    a = ap.parse_args()
    os.environ["MDH_T4_TRACE"] = "1"
    import torch
    import bench
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device
    dev = torch.device("cuda", 0)
    flush = bench.L2Flush(dev)
    for name in a.workloads:
        if name.startswith("mm:"):
            from mdh_workloads import specs as S, gen as G
            M, N, K = (int(v) for v in name[3:].split(","))
            spec, inputs = S.matmul(M, N, K, "bf16"), G.matmul_inputs(M, N, K, "bf16")
        else:
            w = bench.workload(name)
            spec, inputs = w["spec"], w["inputs"]()
        plan = Plan(spec, force_tile=a.force_tile)
        tin = [to_device(x, b["dtype"], dev) for x, b in zip(inputs, spec["inputs"])]
        outs = plan.empty_outputs(dev)
        for rep in range(4):
            flush.zero_()
            torch.cuda.synchronize()
            plan(tin, outs)
            torch.cuda.synchronize()
        tr, ee = Plan.t4_trace()
        if not tr:
            print(json.dumps({"workload": name, "trace": "empty (not the 2-SM kernel?)"}))
            continue
        t0 = min(r[2] for r in tr)
        t_end = max(max(r[3], r[4]) for r in tr)
        units = []
        for u, (sm, pair, a0, a1, e, wf, wa, ts, tp) in enumerate(tr):
            units.append({"u": u, "pair": pair, "sm": sm, "start_us": round((a0 - t0) / 1e3, 2),
                          "mma_us": round((a1 - a0) / 1e3, 2), "epi_done_us": round((e - t0) / 1e3, 2),
                          "wait_full_kcyc": round((wf & 0xffffffff) / 1e3, 1), "wait_acc_kcyc": round(wa / 1e3, 1),
                          "issue_kcyc": round((wf >> 32) / 1e3, 1),
                          "mhz": round((wf >> 32) / ((a1 - a0) / 1e3), 0) if a1 > a0 else None,
                          "seen_us": round((ts - t0) / 1e3, 2) if ts else None,
                          "published_us": round((tp - t0) / 1e3, 2) if tp else None})
        pairs = {}
        for x in units:
            pairs.setdefault(x["pair"], []).append(x)
        busy = sorted(round(sum(y["mma_us"] for y in v), 1) for v in pairs.values())
        ends = sorted(max(y["epi_done_us"] for y in v) for v in pairs.values())
        k0 = min(e[0] for e in ee) if ee else t0
        k1 = max(e[1] for e in ee) if ee else t_end
        print(json.dumps({"workload": name, "kernel_us": round((k1 - k0) / 1e3, 2),
                          "entry_spread_us": round((max(e[0] for e in ee) - k0) / 1e3, 2) if ee else None,
                          "first_mma_after_entry_us": round((t0 - k0) / 1e3, 2),
                          "exit_after_last_epilogue_us": round((k1 - t_end) / 1e3, 2),
                          "span_us": round((t_end - t0) / 1e3, 2), "units": len(units),
                          "pairs": len(pairs), "pair_busy_us_min_med_max": [busy[0], busy[len(busy) // 2], busy[-1]],
                          "pair_end_us_min_med_max": [ends[0], ends[len(ends) // 2], ends[-1]],
                          "wait_full_kcyc_total": round(sum(x["wait_full_kcyc"] for x in units), 1),
                          "mma_us_total": round(sum(x["mma_us"] for x in units), 1)}))
        for x in units:
            print(json.dumps(x))
        del tin, outs, plan
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
