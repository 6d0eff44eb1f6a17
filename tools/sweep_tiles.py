"""Measured tile sweep on B200 → tiles/b200.json (replaces ATF).

    python tools/sweep_tiles.py [--out tiles/b200.json] [--reps 15]

For each (workload, candidate tile override) the step is timed with CUDA events (median of
--reps, L2 flushed between reps); the best candidate per (template, dtype, shape bucket)
is written as a table entry.  Every candidate's median is kept in the "sweep" record.
"""
import argparse
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

T4_WIDE = ["bn=256", "bn=512", "bn=256,split=1", "bn=512,split=1", "bn=512,stages=3", "bn=512,split=1,stages=3"]


# (workload, spec builder kwargs, candidates)
def cases():
    from mdh_workloads import specs as S
    from mdh_workloads import gen as G
    import bench

    def bw(name):                   # a bench workload's spec and seeded inputs
        w = bench.workload(name)
        return w["spec"], w["inputs"]()
    return [
        ("dot_f32_2^20", lambda: (S.dot(1 << 20, "f32"), G.dot_inputs(1 << 20, "f32")),
         [f"split={s}" for s in (64, 128, 148, 256, 296, 512, 592, 1184)]),
        ("dot_f32_2^24", lambda: (S.dot(1 << 24, "f32"), G.dot_inputs(1 << 24, "f32")),
         [f"split={s}" for s in (296, 592, 1184, 2368)]),
        ("dot_f32_2^28", lambda: (S.dot(1 << 28, "f32"), G.dot_inputs(1 << 28, "f32")),
         [f"split={s}" for s in (592, 1184, 2368, 4736)]),
        ("dot_i32_2^20", lambda: (S.dot(1 << 20, "i32"), G.dot_inputs(1 << 20, "i32")),
         [f"split={s}" for s in (64, 128, 148, 256, 296, 512)]),
        *[(f"matvec_f32_{n}", (lambda n=n: (S.matvec(n, n), G.gen_inputs(S.matvec(n, n), 2100, "positive"))),
           ["mode=3", "mode=3,per_thread=3"]) for n in (4096, 8192)],
        ("jacobi3d", lambda: (S.jacobi3d(512, 512, 512), G.jacobi3d_inputs(512, 512, 512)),
         [f"zchunk={z}" for z in (8, 16, 32, 64, 128, 255, 510)]
         # T1 block shapes (bx threads along x), 8 outputs per thread, L2 prefetch hints, and the
         # TMA-staged plane ring — every knob of the 7-point kernel
         + [f"zchunk=8,l2pf=2,per_thread={b}" for b in (64, 128)]
         + ["zchunk=8,l2pf=2", "zchunk=8,l2pf=1", "zchunk=16,l2pf=2", "zchunk=8,vec=8",
            "zchunk=8,stages=3", "zchunk=16,stages=6"]),
        ("gaussian2d", lambda: bw("gaussian2d"),
         [f"zchunk={z}" for z in (8, 12, 16, 20, 24, 32, 48, 64)] + ["zchunk=16,mode=1", "zchunk=32,mode=1"]),
        # T5: records per thread (vec = R), CTAs per SM (stages), DB-loop unroll (bk), split
        ("prl_A", lambda: bw("prl_A"),
         ["split=1", "vec=8", "stages=2", "bk=2", "bk=8", "vec=8,bk=2"]),
        # T3: SGEMM split, the one-CTA-per-SM fragment-pipelined kernel (stages=2), the FFMA form (mode=0)
        ("matmul_f32", lambda: bw("matmul_f32"),
         ["split=1", "split=2", "stages=2", "mode=0", "stages=2,mode=0"]),
        # T6: the streaming scan vs the segmented grid-barrier scan at three segment sizes
        # T6 MBBS: the column fold's row-range splits (default: fill 8 × 256 threads per SM)
        ("mbbs_f32", lambda: bw("mbbs_f32"), [f"split={c}" for c in (4, 6, 7, 8, 9, 10, 12, 16, 24, 32)]),
        ("prefix_sum_f32", lambda: bw("prefix_sum_f32"),
         [f"seg={g}" for g in (65536, 262144, 1048576)]),
        ("prl_B", lambda: (S.prl(1 << 14, 1 << 20), G.prl_inputs(1 << 14, 1 << 20)),
         [f"split={s}" for s in (8, 16, 32, 37, 48, 64)]),
        # T4 2-SM: pair-tile width (256 / 512) × whole tiles vs stream-K for the last wave
        # (wide tiles: ring stages 4 with one epilogue staging buffer, or 3 with two)
        ("t4_mm_bf16_4096", lambda: (S.matmul(4096, 4096, 4096, "bf16"), G.matmul_inputs(4096, 4096, 4096, "bf16", "signed")),
         T4_WIDE),
        ("t4_mm_bf16_8192", lambda: (S.matmul(8192, 8192, 8192, "bf16"), G.matmul_inputs(8192, 8192, 8192, "bf16", "signed")),
         T4_WIDE),
        ("t4_mm_bf16_2048", lambda: (S.matmul(2048, 2048, 2048, "bf16"), G.matmul_inputs(2048, 2048, 2048, "bf16", "signed")),
         T4_WIDE),
        ("t4_mcc_bf16_conv5_1", lambda: (S.mcc(256, 7, 7, 512, 3, 3, 512, "bf16"),
                                         G.mcc_inputs(S.mcc(256, 7, 7, 512, 3, 3, 512, "bf16"))),
         T4_WIDE),
        # per-rank shapes of the strong-scaled configs (bench.py --gpus N):
        # MatMul 4096³ on M at 2/4/8 GPUs, Jacobi3D 512³ z-slabs, PRL A/B DB slices
        *[(f"rank_mm_bf16_{m}", (lambda m=m: (S.matmul(m, 4096, 4096, "bf16"), G.matmul_inputs(m, 4096, 4096, "bf16", "signed"))),
           T4_WIDE + ["bn=256,split=2", "bn=512,split=2", "bn=512,split=2,stages=3"])
          for m in (2048, 1024, 512)],
        *[(f"rank_jacobi3d_{z}", (lambda z=z: (S.jacobi3d(z, 512, 512), G.jacobi3d_inputs(z, 512, 512))),
           [f"zchunk={c},l2pf=2" for c in (3, 4, 5, 6, 7, 8, 10, 12, 16, 32)]) for z in (257, 130, 66)],
        *[(f"rank_prl_A_{i}", (lambda i=i: (S.prl(1 << 20, i), G.prl_inputs(1 << 20, i))),
           [f"split={c}" for c in (1, 2, 3, 4)]) for i in (8192, 4096, 2048)],
        *[(f"rank_prl_B_{i}", (lambda i=i: (S.prl(1 << 14, i), G.prl_inputs(1 << 14, i))),
           [f"split={c}" for c in (9, 18, 27, 37, 48, 64)]) for i in (524288, 262144, 131072)],
        ("mcc_f32_n1", lambda: (S.mcc(1, 7, 7, 512, 3, 3, 512, "f32"),
                                G.mcc_inputs(S.mcc(1, 7, 7, 512, 3, 3, 512, "f32"))),
         [f"split={s}" for s in (1, 8, 16, 32, 64, 72)]),
    ]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "tiles", "b200.json"))
    ap.add_argument("--reps", type=int, default=15)
    ap.add_argument("--only", default=None)
    a = ap.parse_args()
    import torch
    import bench
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device
    dev = torch.device("cuda", 0)
    flush = bench.L2Flush(dev)
    table = json.load(open(a.out)) if os.path.exists(a.out) else {"entries": []}
    entries = {(e["template"], e["dtype"], e.get("f"), e.get("op"), tuple(e["bucket"])): e for e in table.get("entries", [])}
    log = []
    for name, mk, cands in cases():
        if a.only and not any(o in name for o in a.only.split(",")):
            continue
        spec, host = mk()
        tin = None
        res = []
        for c in [None] + cands:
            plan = Plan(spec, force_tile=c) if c else Plan(spec)
            if tin is None:
                tin = [to_device(x, b["dtype"], dev) for x, b in zip(host, spec["inputs"])]
            outs = plan.empty_outputs(dev)
            ws = plan.workspace(dev) if plan.workspace_bytes else None
            step = lambda: plan(tin, outs, workspace_ptr=ws)
            for _ in range(3):
                step()
            torch.cuda.synchronize()
            ts = sorted(bench.time_steps(step, a.reps, torch.cuda.current_stream(), flush))
            med = ts[len(ts) // 2]
            d = plan.describe()
            res.append((med, c, d))
            print(json.dumps({"workload": name, "cand": c or "default", "us": round(med * 1e6, 2),
                              "template": d["template"], "tiles": d["tiles"]}), flush=True)
        best = min(res, key=lambda r: r[0])
        d = best[2]
        if d["template"] in ("T3_simt_contraction", "T4_tcgen05_contraction"):
            c = d["contraction"]
            bucket = [round(math.log2(c["M"]), 2), round(math.log2(c["N"]), 2), round(math.log2(c["K"] * c["Z"]), 2)]
        else:
            bucket = [round(math.log2(d["Ncc"]), 2), round(math.log2(d["Nred"]), 2)]
        dtype = spec["inputs"][0]["dtype"]
        tiles = {}
        if best[1]:
            for kv in best[1].split(","):
                k, v = kv.split("=")
                tiles[k] = int(v)
        else:
            # the default won: record the knobs it resolved to (a table entry of {} would
            # fall back to the template defaults, not to the nearest bucket it was timed with)
            knobs = {"T1_stencil": ("zchunk", "l2pf"), "T2_reduce": ("split",), "T4_tcgen05_contraction": ("bn", "split", "stages"),
                     "T5_prl_pairwise": ("split", "vec", "stages", "bk"), "T3_simt_contraction": ("split",),
                     "T6_prefix_scan": ("seg", "split")}.get(d["template"], ())
            tiles = {k: int(d["tiles"][k]) for k in knobs if k in d["tiles"]}
        fname = spec["f"]
        opcls = next((o for o in spec["ops"] if o == "PS_ADD"), None) or next((o for o in spec["ops"] if o != "CC"), "CC")
        key = (d["template"], dtype, fname, opcls, tuple(bucket))
        entries[key] = {"template": d["template"], "dtype": dtype, "f": fname, "op": opcls, "bucket": bucket, "tiles": tiles,
                        "workload": name, "median_us": round(best[0] * 1e6, 2),
                        "default_us": round(res[0][0] * 1e6, 2),
                        "sweep": {(r[1] or "default"): round(r[0] * 1e6, 2) for r in res}}
        log.append(entries[key])
        del tin
        torch.cuda.empty_cache()
    table["entries"] = sorted(entries.values(), key=lambda e: (e["template"], e["dtype"], e["bucket"]))
    table["comment"] = ("Tile table for libmdh on B200 (sm_100a), produced by tools/sweep_tiles.py: median CUDA-event "
                        "time of every candidate (L2 flushed), best per (template, dtype, log2 shape bucket). "
                        "An entry with empty tiles means the planner default won.")
    with open(a.out, "w") as f:
        json.dump(table, f, indent=1)
    print("wrote", a.out, len(table["entries"]), "entries")


if __name__ == "__main__":
    main()
