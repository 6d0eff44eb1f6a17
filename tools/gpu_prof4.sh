cd $GRAFT_REPO_ROOT
timeout 600 ncu --set full --clock-control none -k regex:gemm2 -s 1 -c 1 -o gpurun_out/prof_gemm2 python tools/time_one.py matmul_bf16 --force-tile cluster=2 --reps 2 > gpurun_out/prof_gemm2.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:gemm_kernel -s 1 -c 1 -o gpurun_out/prof_gemm1 python tools/time_one.py matmul_bf16 --reps 2 > gpurun_out/prof_gemm1.log 2>&1
