cd $GRAFT_REPO_ROOT
timeout 300 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none --csv --log-file gpurun_out/mcc_split.csv python tools/time_one.py mcc_bf16 --reps 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none --csv --log-file gpurun_out/mcc_nosplit.csv python tools/time_one.py mcc_bf16 --reps 3 --force-tile split=1 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none --csv --log-file gpurun_out/mm_split.csv python tools/time_one.py matmul_bf16 --reps 3 > /dev/null 2>&1
