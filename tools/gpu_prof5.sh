cd $GRAFT_REPO_ROOT
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_kernel -s 1 -c 1 -o gpurun_out/prof_mccbox python tools/time_one.py mcc_bf16 --reps 2 > gpurun_out/prof_mccbox.log 2>&1
