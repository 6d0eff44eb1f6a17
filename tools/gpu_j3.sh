cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/j3.txt
: > $o
timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sweeps.py -q -m gpu -x -k "jacobi or sweeps" >> $o 2>&1
for ft in "per_thread=32" "per_thread=64" "per_thread=128" "per_thread=64,zchunk=16" "per_thread=128,zchunk=16" "per_thread=128,zchunk=4" "per_thread=64,zchunk=4"; do
timeout 200 python tools/time_one.py jacobi3d --reps 20 --force-tile $ft 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print('$ft', d['workload'], d['ms'], d['value'], d['frac'])
    except Exception: pass" >> $o
done
cat $o | tail -9
