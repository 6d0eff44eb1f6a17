cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k regex:t3_linear -s 1 -c 1 -f -o gpurun_out/prof_t3 python tools/profile_one.py --workload matmul_f32 --reps 2 > gpurun_out/prof_t3.log 2>&1
ncu -i gpurun_out/prof_t3.ncu-rep --page raw --csv > gpurun_out/prof_t3.raw.csv 2>&1
ls -la gpurun_out/prof_t3*
