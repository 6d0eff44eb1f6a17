cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/mv.txt
: > $o
timeout 300 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "matvec or reductions or dot" >> $o 2>&1; echo "tests rc=$?" >> $o
timeout 200 python tools/time_one.py matvec_f32 matvec_4096 --reps 20 2>&1 | cut -c1-140 >> $o
tail -4 $o
