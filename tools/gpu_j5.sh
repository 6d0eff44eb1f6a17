cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/j5.txt
: > $o
timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sweeps.py -q -m gpu -x -k "jacobi or sweeps" >> $o 2>&1; echo "tests4 rc=$?" >> $o
MDH_FORCE_TILE=vec=8 timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sweeps.py -q -m gpu -x -k "jacobi or sweeps" >> $o 2>&1; echo "tests8 rc=$?" >> $o
for ft in "vec=4" "vec=8" "vec=8,zchunk=16" "vec=8,zchunk=4" "vec=8,per_thread=64"; do
timeout 200 python tools/time_one.py jacobi3d jacobi3d_sweeps8 --reps 20 --force-tile $ft 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print('$ft', d['workload'], d['ms'], d['value'], d['frac'])
    except Exception as e: print(l.strip()[:150])" >> $o
done
grep -v "^\.\|passed" $o | tail -14; grep "rc=" $o
