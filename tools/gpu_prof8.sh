cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ncu --set full --import-source on --clock-control none -k regex:t6_stream -c 1 -o gpurun_out/prof_prefix_stream -f python tools/profile_one.py --workload prefix_sum_f32 --reps 2 > gpurun_out/p8.log 2>&1
ls -la gpurun_out/*.ncu-rep
