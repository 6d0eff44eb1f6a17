# r1h: ncu --set full of the 7-point Jacobi kernel with the L2::256B hint (table default) and
# of the headline wide 2-SM GEMM on this round's fresh box; GPU parity tests for T1
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1h
timeout 300 ncu --set full --clock-control none --import-source on -k regex:t1_j3d7 -s 1 -c 1 -f \
    -o gpurun_out/r1h/prof_jacobi python tools/profile_one.py --workload jacobi3d --reps 2 > gpurun_out/r1h/pj.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:gemm2_kernel -s 1 -c 1 -f \
    -o gpurun_out/r1h/prof_mm python tools/profile_one.py --workload matmul_bf16 --reps 2 > gpurun_out/r1h/pm.log 2>&1
timeout 600 python -m pytest tests -q -m gpu -k "jacobi or stencil or gaussian" > gpurun_out/r1h/t1_tests.log 2>&1
tail -2 gpurun_out/r1h/t1_tests.log; ls gpurun_out/r1h
