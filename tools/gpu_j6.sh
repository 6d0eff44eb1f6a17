cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/j6.txt
: > $o
for rep in 1 2; do
timeout 200 python tools/time_one.py jacobi3d jacobi3d_sweeps8 --reps 20 2>&1 | cut -c1-120 >> $o
done
cat $o
