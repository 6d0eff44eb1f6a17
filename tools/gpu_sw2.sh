cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python tools/time_one.py jacobi3d jacobi3d_sweeps8 --reps 10 2>&1 | cut -c1-200 > gpurun_out/sw2.txt
cat gpurun_out/sw2.txt
