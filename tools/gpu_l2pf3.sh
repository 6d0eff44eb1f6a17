# L2::256B hint on the box-window (Gaussian_2D) loads and the MBBS column fold; interleaved reps
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/l2pf3.txt
: > $o
for rep in 1 2 3; do
timeout 300 python tools/time_one.py gaussian2d mbbs_f32 prefix_sum_f32 jacobi3d --reps 20 2>&1 | cut -c1-110 >> $o
done
timeout 600 python -m pytest tests -q -m gpu -k "gaussian or stencil or box or mbbs or scan or ps or prefix" >> $o 2>&1
cat $o
