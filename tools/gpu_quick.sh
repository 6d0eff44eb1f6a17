# quick GPU check: selected parity tests + timing of selected workloads
# usage: bash tools/gpu_quick.sh "<pytest -k expr>" "<workloads...>"
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x --timeout=240 -k "$1" > gpurun_out/quick_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/quick_tests.log
tail -5 gpurun_out/quick_tests.log
timeout 300 python tools/time_one.py $2 > gpurun_out/quick_time.log 2>&1
cat gpurun_out/quick_time.log | tail -20
