cd $GRAFT_REPO_ROOT
export MDH_DEBUG_SYNC=1
timeout 400 python -m pytest tests/test_gpu_parity.py tests/test_directive.py -q -m gpu -k "tcgen05 or bf16 or mcc or directive or variants" > gpurun_out/t6.txt 2>&1
unset MDH_DEBUG_SYNC
for i in 1 2; do timeout 300 python tools/time_one.py matmul_bf16 mcc_bf16 --reps 20 >> gpurun_out/t6.txt 2>&1; done
timeout 300 python tools/time_one.py matmul_bf16 mcc_bf16 --reps 20 --force-tile split=1 >> gpurun_out/t6.txt 2>&1
