cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/n1.txt
: > $o
for ft in "split=0" "split=4" "split=8" "split=12" "split=18" "implicit=2" "implicit=2,split=8" "implicit=3,split=8"; do
timeout 200 python tools/time_one.py mcc_bf16_n1 --reps 20 --force-tile $ft 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print('$ft', d['workload'], d['ms'], d['value'], d['frac'])
    except Exception as e: print(l.strip()[:150])" >> $o
done
cat $o
