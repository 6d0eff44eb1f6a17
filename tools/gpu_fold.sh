cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/fold.txt
: > $o
MDH_DEBUG_SYNC=1 timeout 400 python -m pytest tests/test_gpu_parity.py -q -m gpu -x --timeout=200 -k "stream_k or im2col or mcc or matmul_bf16" >> $o 2>&1; echo "tests rc=$?" >> $o
timeout 200 python tools/time_one.py matmul_bf16 mcc_bf16 mm:12544,512,4608 mm:8192,8192,8192 --reps 20 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print(d['workload'], d['ms'], d['value'], d['frac'])
    except Exception: print(l.strip()[:200])" >> $o
timeout 200 python tools/t4_trace.py mcc_bf16 matmul_bf16 > gpurun_out/trace_fold.jsonl 2>&1
grep span gpurun_out/trace_fold.jsonl | cut -c1-330 >> $o
tail -9 $o
