cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1f
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/wbw tools/wbw_probe.cu && /tmp/wbw > gpurun_out/r1f/wbw.log 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:gemm_kernel -s 1 -c 1 -f \
    -o gpurun_out/r1f/prof_ccsd_bf16 python tools/profile_one.py --workload ccsd_bf16 --reps 2 > gpurun_out/r1f/ccsd.log 2>&1
cat gpurun_out/r1f/wbw.log
