cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/t3b.txt
: > $o
timeout 300 python tools/time_spec.py "S.ccsd_sd2()" "S.mcc(1, 7, 7, 512, 3, 3, 512, 'f32')" "S.mcc(16, 7, 7, 512, 3, 3, 512, 'f32')" "S.bmatmul(16, 10, 500, 64, 'f32')" "S.matmul_t(1024, 1024, 1024, 'f32')" >> $o 2>&1
timeout 300 python tools/time_one.py matmul_f32 --reps 10 >> $o 2>&1
timeout 400 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "f32 or fig3 or int32 or ccsd or mcc or matmul" >> $o 2>&1; echo "tests rc=$?" >> $o
tail -9 $o | cut -c1-200
