cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_sweeps.py tests/test_gpu_parity.py -q -m gpu -x -k "sweeps or jacobi" > gpurun_out/sw3.txt 2>&1
timeout 300 python tools/time_one.py jacobi3d jacobi3d_sweeps8 --reps 10 2>&1 | cut -c1-160 >> gpurun_out/sw3.txt
tail -4 gpurun_out/sw3.txt
