cd $GRAFT_REPO_ROOT
export MDH_DEBUG_SYNC=1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -rf -x -k "tcgen05 and mnk0" > gpurun_out/t4_first.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -rf -k "tcgen05 or bf16_full" > gpurun_out/t4_tests.txt 2>&1
unset MDH_DEBUG_SYNC
timeout 300 python bench.py --no-suite --no-cpu-baseline > gpurun_out/t4_bench.json 2> gpurun_out/t4_bench.err
echo done
