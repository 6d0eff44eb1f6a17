cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/ab.txt
: > $o
for rep in 1 2 3; do
for ft in "bn=256" "bn=512" "bn=512,split=1" "bn=256,split=1"; do
timeout 200 python tools/time_one.py matmul_bf16 --reps 30 --force-tile $ft 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print('$ft', d['workload'], d['ms'], d['value'])
    except Exception: pass" >> $o
done
done
cat $o
