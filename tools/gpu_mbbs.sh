cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/mbbs.txt
MDH_DEBUG_SYNC=1 timeout 400 python -m pytest tests/test_ps_operator.py -q -m gpu -x --timeout=200 > $o 2>&1; echo "tests rc=$?" >> $o
timeout 200 python tools/time_one.py mbbs_f32 prefix_sum_f32 --reps 20 2>&1 | cut -c1-160 >> $o
tail -5 $o
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv python tools/profile_one.py --workload mbbs_f32 --reps 2 > gpurun_out/mbbs_ncu.csv 2>&1
