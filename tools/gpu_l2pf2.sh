# after: Jacobi default l2pf=2 from the table; T2 loads with the L2::256B hint
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/l2pf2.txt
: > $o
for rep in 1 2; do
timeout 300 python tools/time_one.py jacobi3d jacobi3d_sweeps8 matvec_f32 matvec_4096 dot_f32 dot_i32 dot_f32_2^28 --reps 20 2>&1 | cut -c1-110 >> $o
done
timeout 600 python -m pytest tests -q -m gpu -k "stencil or jacobi or dot or matvec or reduce or t2" >> $o 2>&1
cat $o
