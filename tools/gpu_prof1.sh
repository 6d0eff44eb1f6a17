cd $GRAFT_REPO_ROOT
NCU=ncu
$NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_matmul_bf16.csv python bench.py --steps 2 --warmup 3 --no-suite --no-cpu-baseline > gpurun_out/launches_bench.log 2>&1
for w in matmul_bf16 jacobi3d dot_f32_2^28 prl_A matvec_f32 matmul_f32; do
  k=".*"
  timeout 600 $NCU --set full --clock-control none --import-source on -s 1 -c 1 -o gpurun_out/prof_$w python tools/profile_one.py --workload $w --reps 2 > gpurun_out/prof_$w.log 2>&1
done
echo done
