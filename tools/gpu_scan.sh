cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/scan.txt
: > $o
MDH_DEBUG_SYNC=1 timeout 400 python -m pytest tests/test_ps_operator.py -q -m gpu -x >> $o 2>&1; echo "tests rc=$?" >> $o
for rep in 1 2; do timeout 200 python tools/time_one.py prefix_sum_f32 --reps 20 2>&1 | cut -c1-130 >> $o; done
tail -4 $o
