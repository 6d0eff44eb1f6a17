"""Context measurement only (not a product path): cuBLAS bf16 GEMM throughput, CUDA
events, L2 flushed, same protocol as bench.py.

    python tools/cublas_ref.py [M,N,K ...]      (default: 4096³ and 8192³)
"""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench

dev = torch.device("cuda", 0)
flush = bench.L2Flush(dev)
shapes = [tuple(int(v) for v in s.split(",")) for s in sys.argv[1:]] or [(4096,) * 3, (8192,) * 3]
for M, N, K in shapes:
    a = torch.randn(M, K, device=dev, dtype=torch.bfloat16)
    b = torch.randn(K, N, device=dev, dtype=torch.bfloat16)
    for out in ("bf16", "f32"):
        if out == "bf16":
            fn = lambda: torch.matmul(a, b)
        else:
            c = torch.empty(M, N, device=dev, dtype=torch.float32)
            fn = lambda: torch.matmul(a, b, out_dtype=torch.float32)
        try:
            for _ in range(5):
                fn()
            torch.cuda.synchronize()
        except Exception as e:  # out_dtype needs a recent torch
            print(json.dumps({"cublas": [M, N, K], "out": out, "error": str(e)[:100]}))
            continue
        ts = sorted(bench.time_steps(fn, 20, torch.cuda.current_stream(), flush))
        med = ts[len(ts) // 2]
        print(json.dumps({"cublas": [M, N, K], "out": out, "ms": round(med * 1e3, 4),
                          "TFLOP/s": round(2 * M * N * K / med / 1e12, 1)}), flush=True)
