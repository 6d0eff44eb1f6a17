cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/sweeps.txt
: > $o
MDH_DEBUG_SYNC=1 timeout 400 python -m pytest tests/test_gpu_sweeps.py tests/test_gpu_parity.py -q -m gpu -x --timeout=200 -k "sweeps or jacobi" >> $o 2>&1; echo "tests rc=$?" >> $o
tail -5 $o
