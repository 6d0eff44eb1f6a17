# full GPU round (final round-1 record): tests, smoke, bench (+ reference arm), ncu launch list of the bench
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1k
timeout 1200 python -m pytest tests -q -m gpu > gpurun_out/r1k/tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r1k/tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/r1k/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/r1k/bench.json 2> gpurun_out/r1k/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r1k/ref.json 2> gpurun_out/r1k/ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r1k/launches.csv python bench.py --steps 2 --warmup 3 --no-suite --no-cpu-baseline > gpurun_out/r1k/ncu_bench.log 2>&1
tail -3 gpurun_out/r1k/tests.log; tail -2 gpurun_out/r1k/smoke.log
