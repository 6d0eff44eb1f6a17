# one ncu --set full capture per §8 workload's dominant kernel + the bench launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1d
cap() {  # name kernel-regex
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$2 -s 1 -c 1 -f \
    -o gpurun_out/r1d/prof_$1 python tools/profile_one.py --workload $1 --reps 3 > gpurun_out/r1d/$1.log 2>&1
}
cap matmul_bf16 gemm2_kernel
cap mcc_bf16 gemm_kernel
cap ccsd_bf16 gemm_kernel
cap matmul_f32 t3_
cap jacobi3d t1_
ls gpurun_out/r1d
