"""Context measurement only (not a product path): PyTorch/cuBLAS library kernels for the
HBM-bound suite entries, same protocol as bench.py (CUDA events, L2 flushed before every
step, median of the timed steps).  Shows how much of a small workload's time is the
protocol's cold-start floor (launch, L2/TLB refill) rather than the kernel.

    python tools/lib_ref_hbm.py
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench

dev = torch.device("cuda", 0)
flush = bench.L2Flush(dev)
g = torch.Generator(device=dev).manual_seed(7)


def run(name, fn, nbytes):
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    ts = sorted(bench.time_steps(fn, 20, torch.cuda.current_stream(), flush))
    sec = ts[len(ts) // 2]
    print(json.dumps({"lib": name, "ms": round(sec * 1e3, 4), "GB/s": round(nbytes / sec / 1e9, 1)}))


n = 1 << 20
x = torch.rand(n, device=dev, generator=g)
y = torch.rand(n, device=dev, generator=g)
run("torch.dot fp32 2^20", lambda: torch.dot(x, y), 8 * n)
xi = torch.randint(0, 100, (n,), device=dev, dtype=torch.int32)
yi = torch.randint(0, 100, (n,), device=dev, dtype=torch.int32)
run("torch (x*y).sum int32 2^20", lambda: (xi * yi).sum(), 8 * n)
n28 = 1 << 28
a = torch.rand(n28, device=dev, generator=g)
b = torch.rand(n28, device=dev, generator=g)
run("torch.dot fp32 2^28", lambda: torch.dot(a, b), 8 * n28)
del a, b
A = torch.rand(8192, 8192, device=dev, generator=g)
v = torch.rand(8192, device=dev, generator=g)
run("torch.mv fp32 8192^2", lambda: torch.mv(A, v), 4 * 8192 * 8192 + 8 * 8192)
run("torch.cumsum(A.sum(0)) fp32 8192^2 (MBBS)", lambda: torch.cumsum(A.sum(0), 0), 4 * 8192 * 8192)
del A
p = torch.rand(1 << 26, device=dev, generator=g)
run("torch.cumsum fp32 2^26", lambda: torch.cumsum(p, 0), 8 * (1 << 26))
