# final round-1 captures: ncu --set full of the headline kernel (MatMul 4096^3, wide whole tiles),
# MCC conv5_1, the SGEMM, the MBBS column fold; the bench launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1f
cap() {  # name kernel-regex
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$2 -s 1 -c 1 -f \
    -o gpurun_out/r1f/prof_$1 python tools/profile_one.py --workload $1 --reps 3 > gpurun_out/r1f/$1.log 2>&1
}
cap matmul_bf16 gemm2_kernel
cap mcc_bf16 gemm2_kernel
cap matmul_f32 t3_linear
cap mbbs_f32 t6_colfold
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r1f/launches_bench.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/r1f/bench_under_ncu.log 2>&1
ls -la gpurun_out/r1f
