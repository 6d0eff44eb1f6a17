# A/B: L2 prefetch-size hint on the 7-point Jacobi row loads (tile knob l2pf; values 3/4 were a z-pipelined variant, since removed), same box, interleaved
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/l2pf.txt
: > $o
for rep in 1 2 3; do
for t in zchunk=8 zchunk=8,l2pf=1 zchunk=8,l2pf=2 zchunk=8,l2pf=3 zchunk=8,l2pf=4 zchunk=16,l2pf=4; do
echo -n "$t " >> $o
timeout 200 python tools/time_one.py jacobi3d jacobi3d_sweeps8 --reps 20 --force-tile $t 2>&1 | cut -c1-120 | tr '\n' ' ' >> $o
echo >> $o
done
done
timeout 300 python -m pytest tests -q -m gpu -k "stencil or jacobi" >> $o 2>&1
cat $o
