"""Context measurement only (not a product path): cuDNN bf16 conv2d for the MCC layer
(conv5_1 3x3/s2, C=K=512, N=256, NHWC), CUDA events, L2 flushed, same protocol as bench.py."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench

dev = torch.device("cuda", 0)
flush = bench.L2Flush(dev)
torch.backends.cudnn.benchmark = True
N = int(sys.argv[1]) if len(sys.argv) > 1 else 256
x = torch.rand(N, 512, 16, 16, device=dev, dtype=torch.bfloat16).to(memory_format=torch.channels_last)
w = torch.randn(512, 512, 3, 3, device=dev, dtype=torch.bfloat16).to(memory_format=torch.channels_last)
fn = lambda: torch.nn.functional.conv2d(x, w, stride=2)
for _ in range(10):
    fn()
torch.cuda.synchronize()
ts = sorted(bench.time_steps(fn, 20, torch.cuda.current_stream(), flush))
med = ts[len(ts) // 2]
print(json.dumps({"cudnn_conv5_1": N, "ms": round(med * 1e3, 4), "TFLOP/s": round(2 * N * 49 * 512 * 4608 / med / 1e12, 1)}))
