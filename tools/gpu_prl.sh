cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/prl.txt
: > $o
for ft in "split=0" "split=2" "split=3" "split=6"; do
timeout 200 python tools/time_one.py prl_A --reps 5 --force-tile $ft 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print('$ft', d['workload'], d['ms'], d['value'], d['frac'], d['tiles']['split'])
    except Exception as e: print(l.strip()[:150])" >> $o
done
cat $o
