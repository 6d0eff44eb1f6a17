cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/t4h.txt
: > $o
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_directive.py -q -m gpu -x --timeout=200 >> $o 2>&1; echo "parity tests rc=$?" >> $o
timeout 200 python tools/time_one.py matmul_bf16 mcc_bf16 ccsd_bf16 mcc_caps_bf16 mm:8192,8192,8192 --reps 20 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print(d['workload'], d['ms'], d['value'], d['frac'], d['tiles']['bn'], d['tiles']['cluster'])
    except Exception: print(l.strip()[:200])" >> $o
tail -9 $o
