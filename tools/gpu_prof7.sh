cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export MDH_FORCE_TILE=seg=16777216
timeout 300 ncu --set full --clock-control none -k regex:t6_seg -c 1 -o gpurun_out/prof_prefix_sum_f32 -f python tools/profile_one.py --workload prefix_sum_f32 --reps 2 > gpurun_out/p7a.log 2>&1
unset MDH_FORCE_TILE
timeout 300 ncu --set full --clock-control none -k regex:t6_fold -c 1 -o gpurun_out/prof_mbbs_f32 -f python tools/profile_one.py --workload mbbs_f32 --reps 2 > gpurun_out/p7b.log 2>&1
ls -la gpurun_out/*.ncu-rep
