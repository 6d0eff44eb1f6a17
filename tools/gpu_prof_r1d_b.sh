# one ncu --set full capture per §8 workload's dominant kernel + the bench launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1d
cap() {  # name kernel-regex
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$2 -s 1 -c 1 -f \
    -o gpurun_out/r1d/prof_$1 python tools/profile_one.py --workload $1 --reps 3 > gpurun_out/r1d/$1.log 2>&1
}
cap dot_f32_2^28 t2_
cap matvec_f32 t2_
cap prl_A t5_kernel
cap prl_B t5_kernel
cap prefix_sum_f32 t6_stream
cap mbbs_f32 t6_fold
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r1d/launches_bench.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/r1d/bench_under_ncu.log 2>&1
ls gpurun_out/r1d
