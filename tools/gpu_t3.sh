cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/t3.txt
: > $o
for rep in 1 2; do
for ft in "per_thread=1" "per_thread=2"; do
timeout 200 python tools/time_one.py matmul_f32 --reps 10 --force-tile $ft 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print('$ft', d['workload'], d['ms'], d['value'], d['frac'])
    except Exception as e: print(l.strip()[:150])" >> $o
done
done
MDH_FORCE_TILE=per_thread=2 timeout 300 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "matmul and f32 or fig3" >> $o 2>&1; echo "tests rc=$?" >> $o
tail -8 $o
