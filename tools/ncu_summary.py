"""Summarise ncu reports (.ncu-rep) into profiles/<round>_ncu_summary.md and
profiles/ncu_traffic.json (DRAM bytes per launch, read by bench.py's roofline.traffic).

    python tools/ncu_summary.py --round r1 gpurun_out/prof_*.ncu-rep [--launches gpurun_out/launches_*.csv]
"""
import argparse
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_%peak"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_%peak"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor_pipe_%"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_active_%"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occupancy_%"),
    ("lts__t_sector_hit_rate.pct", "L2_hit_%"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-9, "us": 1e-6,
              "usecond": 1e-6, "msecond": 1e-3, "ms": 1e-3, "nsecond": 1e-9, "second": 1.0}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return []
    h, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[h.index("Kernel Name")]}
        for m, short in METRICS:
            if m in h:
                i = h.index(m)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    v = r[i]
                if isinstance(v, float) and units[i] in UNIT_SCALE:
                    v = v * UNIT_SCALE[units[i]]
                d[short] = v
        res.append(d)
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", default="r1")
    ap.add_argument("--launches", nargs="*", default=[])
    ap.add_argument("reps", nargs="+")
    a = ap.parse_args()
    lines = [f"# ncu summary — round {a.round}", "",
             "One `ncu --set full --clock-control none` capture per workload (tools/profile_one.py), "
             "kernel-level metrics read with `ncu -i … --page raw --csv`. Times under ncu are cold-cache and "
             "serialised; compare shares and counters, not absolutes.", "",
             "| workload | kernel | duration (us) | DRAM read (MB) | DRAM write (MB) | DRAM %peak | SM %peak | "
             "tensor pipe % | issue active % | occupancy % | L2 hit % | regs | grid×block |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    traffic_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    for rep in a.reps:
        wl = os.path.basename(rep).replace(".ncu-rep", "").split("_", 1)[1]
        for d in raw(rep):
            f = lambda k, s=1.0, p=1: (f"{d[k] / s:.{p}f}" if isinstance(d.get(k), float) else str(d.get(k, "")))
            lines.append(f"| {wl} | `{d['kernel'][:60]}` | {f('duration', 1e-6)} | {f('dram_read', 1e6)} | "
                         f"{f('dram_write', 1e6)} | {f('dram_%peak')} | {f('sm_%peak')} | {f('tensor_pipe_%')} | "
                         f"{f('issue_active_%')} | {f('occupancy_%')} | {f('L2_hit_%')} | {f('regs', 1, 0)} | "
                         f"{f('grid', 1, 0)}×{f('block', 1, 0)} |")
            if isinstance(d.get("dram_read"), float):
                traffic[wl] = d["dram_read"] + d.get("dram_write", 0.0)
    for lf in a.launches:
        lines += ["", f"## launch list `{os.path.basename(lf)}` (gpu__time_duration per launch)", ""]
        rows = [r for r in csv.reader(open(lf)) if len(r) > 14 and r[0].isdigit()]
        tot = {}
        for r in rows:
            tot.setdefault(r[4][:70], []).append(float(r[14]))
        allt = sum(sum(v) for v in tot.values())
        lines.append("| kernel | launches | mean (us) | share of listed time |")
        lines.append("|---|---|---|---|")
        for k, v in sorted(tot.items(), key=lambda kv: -sum(kv[1])):
            lines.append(f"| `{k}` | {len(v)} | {sum(v) / len(v) / 1e3:.2f} | {sum(v) / allt:.1%} |")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", f"{a.round}_ncu_summary.md"), "w") as fh:
        fh.write("\n".join(lines) + "\n")
    with open(traffic_path, "w") as fh:
        json.dump(traffic, fh, indent=1, sort_keys=True)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
