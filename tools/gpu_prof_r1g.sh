cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1g
timeout 300 ncu --set full --clock-control none --import-source on -k regex:gemm2_kernel -s 1 -c 1 -f \
    -o gpurun_out/r1g/prof_mcc_ic python tools/profile_one.py --workload mcc_bf16 --reps 2 > gpurun_out/r1g/mcc.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:gemm2_kernel -s 1 -c 1 -f \
    -o gpurun_out/r1g/prof_mm python tools/profile_one.py --workload matmul_bf16 --reps 2 > gpurun_out/r1g/mm.log 2>&1
ls gpurun_out/r1g
