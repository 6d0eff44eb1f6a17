cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q -rf --timeout 600 > gpurun_out/run3_tests.txt 2>&1
for i in 1 2; do timeout 200 python tools/time_one.py matmul_bf16 --reps 20 >> gpurun_out/run3_mm.txt 2>&1; timeout 200 python tools/time_one.py matmul_bf16 --reps 20 --force-tile cluster=2 >> gpurun_out/run3_mm.txt 2>&1; done
timeout 900 python bench.py > gpurun_out/run3_bench.json 2> gpurun_out/run3_bench.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/run3_smoke.txt 2>&1
