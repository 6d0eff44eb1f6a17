cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/t3c.txt
: > $o
timeout 300 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "matmul and f32 or fig3 or matvec" >> $o 2>&1; echo "tests rc=$?" >> $o
for rep in 1 2; do
timeout 200 python tools/time_one.py matmul_f32 --reps 10 2>&1 | cut -c1-140 >> $o
timeout 200 python tools/time_one.py matmul_f32 --reps 10 --force-tile stages=1 2>&1 | cut -c1-140 >> $o
done
tail -6 $o
