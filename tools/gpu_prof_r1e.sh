# ncu --set full captures of the 2-SM T4 kernel (MatMul headline, MCC) + the bench launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1e
cap() {  # name kernel-regex
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$2 -s 1 -c 1 -f \
    -o gpurun_out/r1e/prof_$1 python tools/profile_one.py --workload $1 --reps 3 > gpurun_out/r1e/$1.log 2>&1
}
cap matmul_bf16 gemm2_kernel
cap mcc_bf16 gemm2_kernel
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r1e/launches_bench.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/r1e/bench_under_ncu.log 2>&1
ls -la gpurun_out/r1e
