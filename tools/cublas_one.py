"""Run cuBLAS bf16 GEMM M,N,K a few times (for an ncu capture of its kernel; context only)."""
import sys
import torch
M, N, K = (int(v) for v in (sys.argv[1] if len(sys.argv) > 1 else "4096,4096,4096").split(","))
a = torch.randn(M, K, device="cuda", dtype=torch.bfloat16)
b = torch.randn(K, N, device="cuda", dtype=torch.bfloat16)
for _ in range(4):
    c = a @ b
torch.cuda.synchronize()
