cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/xf.txt
: > $o
MDH_DEBUG_SYNC=1 timeout 500 python -m pytest tests/test_gpu_parity.py -q -m gpu -x --timeout=200 -k "few_tile or mcc or matmul_bf16_tcgen05 or split_tail" >> $o 2>&1; echo "tests rc=$?" >> $o
for ft in "split=0" "split=4" "split=8" "split=18" "split=1"; do
timeout 200 python tools/time_one.py mcc_bf16_n1 --reps 20 --force-tile $ft 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print('$ft', d['workload'], d['ms'], d['value'], d['frac'])
    except Exception as e: print(l.strip()[:150])" >> $o
done
tail -8 $o
