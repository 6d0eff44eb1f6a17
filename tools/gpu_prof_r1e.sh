# r1e: CCSD(T) + MCC full captures with source, and a write-bandwidth ceiling probe
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1e
python - > gpurun_out/r1e/writebw.log 2>&1 <<'PY'
import torch
x = torch.empty(5159780352, dtype=torch.float32, device="cuda")
for _ in range(3): x.fill_(1.0)
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
ts = []
for _ in range(5):
    s.record(); x.fill_(2.0); e.record(); e.synchronize(); ts.append(s.elapsed_time(e))
print("fill 20.6GB ms", ts, "GB/s", 4 * x.numel() / (min(ts) * 1e-3) / 1e9)
PY
cap() {  # name kernel-regex
  timeout 400 ncu --set full --clock-control none --import-source on -k regex:$2 -s 1 -c 1 -f \
    -o gpurun_out/r1e/prof_$1 python tools/profile_one.py --workload $1 --reps 2 > gpurun_out/r1e/$1.log 2>&1
}
cap ccsd_bf16 gemm_kernel
cap mcc_bf16 gemm_kernel
ls -la gpurun_out/r1e
