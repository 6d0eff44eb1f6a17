"""Size-dependent HBM floor under the bench protocol (context for the F-row fractions, not
a product path): torch's copy_ (read + write) and sum (read only) of N fp32 elements,
median of CUDA-event pairs with the L2 flushed before each, as GB/s and as a fraction of
MEASURED_PEAKS.json's copy bandwidth.

    python tools/floor_probe.py 26 28      # log2 N
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import bench
    dev = torch.device("cuda", 0)
    flush = bench.L2Flush(dev)
    pk = bench.peaks()
    st = torch.cuda.current_stream()
    for lg in [int(v) for v in sys.argv[1:]]:
        n = 1 << lg
        a = torch.rand(n, device=dev)
        b = torch.empty_like(a)
        s = torch.empty((), device=dev)
        for name, step, nbytes in (("copy", lambda: b.copy_(a), 8 * n), ("sum", lambda: torch.sum(a, dim=0, out=s), 4 * n)):
            for _ in range(3):
                step()
            ts = sorted(bench.time_steps(step, 15, st, flush))
            med = ts[len(ts) // 2]
            gbs = nbytes / med / 1e9
            print(json.dumps({"probe": name, "log2n": lg, "us": round(med * 1e6, 2), "GB/s": round(gbs, 1),
                              "frac": round(gbs / pk["hbm_gbs"], 4)}), flush=True)
        del a, b
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
