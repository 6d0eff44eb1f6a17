# T4 few-tile split-K: the fold launched as a programmatic dependent of the GEMM
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/xf2.txt
: > $o
timeout 900 python -m pytest tests -q -m gpu -k "mcc or split or t4 or matmul or ccsd" >> $o 2>&1
for rep in 1 2 3; do
timeout 300 python tools/time_one.py mcc_bf16_n1 mcc_bf16 matmul_bf16 --reps 20 2>&1 | cut -c1-110 >> $o
done
timeout 300 compute-sanitizer --tool memcheck python tools/profile_one.py --workload mcc_bf16_n1 --reps 1 2>&1 | tail -2 >> $o
cat $o
