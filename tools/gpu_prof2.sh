cd $GRAFT_REPO_ROOT
for w in ccsd_bf16 mcc_bf16; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_kernel -s 1 -c 1 -o gpurun_out/prof_$w python tools/profile_one.py --workload $w --reps 2 > gpurun_out/prof_$w.log 2>&1
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_mcc.csv python tools/profile_one.py --workload mcc_bf16 --reps 3 > /dev/null 2>&1
echo done
