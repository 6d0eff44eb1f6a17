"""Context measurement only (not a product path): cuBLAS bf16 GEMM throughput at the
headline shape, CUDA events, L2 flushed, same protocol as bench.py."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench

dev = torch.device("cuda", 0)
flush = bench.L2Flush(dev)
for n in (4096, 8192):
    a = torch.randn(n, n, device=dev, dtype=torch.bfloat16)
    b = torch.randn(n, n, device=dev, dtype=torch.bfloat16)
    for _ in range(5):
        c = a @ b
    torch.cuda.synchronize()
    ts = sorted(bench.time_steps(lambda: torch.matmul(a, b), 20, torch.cuda.current_stream(), flush))
    med = ts[len(ts) // 2]
    print(json.dumps({"cublas_bf16_out_bf16": n, "ms": med * 1e3, "TFLOP/s": 2 * n ** 3 / med / 1e12}))
