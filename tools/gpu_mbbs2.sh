cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,launch__grid_size --clock-control none --csv python tools/profile_one.py --workload mbbs_f32 --reps 2 > gpurun_out/mbbs_ncu.csv 2>&1
grep -v "^==" gpurun_out/mbbs_ncu.csv | cut -c1-250 | tail -20
