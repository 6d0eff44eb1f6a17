# full GPU round: tests, smoke, bench (+ reference arm), ncu launch list of the bench
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -q -m gpu > gpurun_out/round_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/round_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/round_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/round_bench.json 2> gpurun_out/round_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/round_ref.json 2> gpurun_out/round_ref.err
tail -3 gpurun_out/round_tests.log; cat gpurun_out/round_smoke.log | tail -2
