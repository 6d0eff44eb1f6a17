"""Small instances of every template, run under compute-sanitizer by tests/test_sanitizer.py
(memcheck / racecheck / synccheck / initcheck on small shapes).

    compute-sanitizer --tool memcheck python tools/sanitize_cases.py [name]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def cases():
    from mdh_workloads import gen as G
    from mdh_workloads import specs as S
    return {
        "t0": (lambda: S.make_spec("t0", ["a", "b", "c"], [9, 5, 7], ["CC", "PW_ADD", "PW_ADD"], "IDENTITY",
                                   [S.buffer("x", "f32", [["a", "c", "b"]], ["a", "b", "c"])],
                                   [S.buffer("y", "f32", [["a"]], ["a", "b", "c"])]), "positive", None),
        "t1": (lambda: S.jacobi3d(18, 21, 133), "positive", None),
        "t2_row": (lambda: S.dot(100003, "f32"), "positive", None),
        "t2_warp": (lambda: S.matvec(1300, 777), "positive", None),
        "t2_col": (lambda: S.reduce_spec([1000, 37], [0]), "positive", None),
        "t3": (lambda: S.matmul(130, 129, 70), "positive", None),
        "t3_lin": (lambda: S.matmul(256, 384, 96), "positive", None),
        "t4": (lambda: S.matmul(300, 264, 200, "bf16"), "positive", None),
        "t4_2sm": (lambda: S.matmul(512, 512, 256, "bf16"), "positive", None),
        "t4_gather": (lambda: S.ccsd_sd1(2, 3, "bf16"), "signed", None),
        "t4_split": (lambda: S.matmul(1280, 768, 512, "bf16"), "positive", "split=3"),
        "t4_ag": (lambda: S.mcc(4, 7, 7, 64, 3, 3, 16, "bf16"), "positive", None),
        "t4_split1": (lambda: S.matmul(2500, 2000, 512, "bf16", out_dtype="bf16"), "positive", "split=2"),
        "t4_sk": (lambda: S.matmul(512, 512, 2048, "bf16"), "positive", "split=2"),
        "t4_wide_sk": (lambda: S.matmul(512, 1024, 1024, "bf16"), "positive", "bn=512,split=2"),
        "t4_wide": (lambda: S.matmul(700, 1000, 512, "bf16"), "positive", "bn=512,split=1"),
        "t4_xfold": (lambda: S.matmul(100, 300, 2048, "bf16"), "positive", None),
        "t4_im2col": (lambda: S.mcc(4, 7, 7, 512, 3, 3, 512, "bf16"), "positive", None),
        "t4_cl4": (lambda: S.matmul(700, 1000, 512, "bf16"), "positive", "cluster=4"),
        "t1_sweep": (lambda: S.jacobi3d_sweep(12, 10, 70), "positive", None),
        "t4_ag4": (lambda: S.mcc_caps(2, 5, 3, 4, 3, 3, 3, dtype="bf16"), "positive", None),
        "t4_conv": (lambda: S.mcc(3, 17, 19, 64, 7, 7, 3, "bf16"), "positive", None),
        "t4_conv_ns3": (lambda: S.mcc(3, 17, 19, 64, 7, 7, 3, "bf16"), "positive", "stages=3"),
        "t4_conv3x3": (lambda: S.mcc(2, 20, 21, 64, 3, 3, 3, "bf16"), "positive", None),
        "t6_colfold": (lambda: S.mbbs(300, 1000), "positive", None),
        "t5": (lambda: S.prl(300, 2000), "prl", None),
        "t6": (lambda: S.prefix_sum([3, 9000], 1), "positive", None),
        "combine": (lambda: S.dot(5000, "i32"), "virtual", None),
    }


def run(name):
    import numpy as np
    import torch
    from mdh_workloads import gen as G
    from paper_conf_sc_schulzegr25_b200 import Plan, to_device, VIRTUAL_SHARD
    from gpu_util import assert_close_full, run_gpu
    mk, kind, tile = cases()[name]
    spec = mk()
    if kind == "prl":
        x = G.prl_inputs(spec["sizes"][0], spec["sizes"][1], seed_base=5800)
    elif kind == "virtual":
        x = G.dot_inputs(5000, "i32")
        parts = []
        for r in range(3):
            p = Plan(spec, world_size=3, rank=r, flags=VIRTUAL_SHARD)
            tin = []
            for b, arr in enumerate(x):
                shp, off, _ = p.local_shape(False, b)
                tin.append(to_device(np.ascontiguousarray(arr[off[0]:off[0] + shp[0]]), "i32", "cuda"))
            outs = p.empty_outputs()
            p(tin, outs)
            parts.append((p, outs))
        parts[0][0].combine_partials([o for _, o in parts])
        torch.cuda.synchronize()
        print(name, "ok")
        return
    else:
        x = G.gen_inputs(spec, 9000, kind)
    got, p = run_gpu(spec, x, force_tile=tile)
    print(name, p.template, "ok")


if __name__ == "__main__":
    names = sys.argv[1:] or list(cases())
    for n in names:
        run(n)
