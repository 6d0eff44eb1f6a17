cd $GRAFT_REPO_ROOT
export MDH_DEBUG_SYNC=1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -rf -k "ccsd_bf16 or mcc_bf16 or matvec or jacobi or dot" > gpurun_out/run2_tests.txt 2>&1
unset MDH_DEBUG_SYNC
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/run2_bench.json 2> gpurun_out/run2_bench.err
echo done
