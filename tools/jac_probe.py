"""Probe the TMA-staged 7-point kernel on one shape / tile string in a fresh process.

    python tools/jac_probe.py Z Y X tile
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def main():
    Z, Y, X = (int(v) for v in sys.argv[1:4])
    tile = sys.argv[4]
    import numpy as np
    from mdh_workloads import gen as G
    from mdh_workloads import specs as S
    from gpu_util import run_gpu
    spec = S.jacobi3d(Z, Y, X)
    x = G.jacobi3d_inputs(Z, Y, X)
    got, p = run_gpu(spec, x, force_tile=tile)
    ref, _ = run_gpu(spec, x, force_tile="stages=0")
    print("ok" if np.array_equal(got[0], ref[0]) else "MISMATCH", Z, Y, X, tile,
          float(np.nanmax(np.abs(got[0] - ref[0]))))


if __name__ == "__main__":
    main()
