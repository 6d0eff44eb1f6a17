"""Run the conv1 N=256 plan with a forced tile string and check 2000 sampled outputs
against the oracle (probe for the small-K direct kernel's staging ring).

    python tools/conv_probe.py stages=3 [N]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def main():
    tile = sys.argv[1] if len(sys.argv) > 1 else None
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 256
    from mdh_workloads import gen as G
    from mdh_workloads import specs as S
    from gpu_util import assert_close_points, run_gpu
    spec = S.mcc(n, 112, 112, 64, 7, 7, 3, "bf16")
    x = G.mcc_inputs(spec)
    got, p = run_gpu(spec, x, force_tile=tile)
    assert_close_points(spec, x, got, 1e-2, n=2000, kind="scale")
    print("ok", tile, n, p.describe()["tiles"]["stages"])


if __name__ == "__main__":
    main()
