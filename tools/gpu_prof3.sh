cd $GRAFT_REPO_ROOT
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_kernel -s 1 -c 1 -o gpurun_out/prof_ccsd2 python tools/profile_one.py --workload ccsd_bf16 --reps 2 > gpurun_out/prof_ccsd2.log 2>&1
echo done
