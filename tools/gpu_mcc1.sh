# MCC diagnosis: A-operand variants, the same M/N/K as a plain GEMM, cuBLAS context
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/mcc1.txt
: > $o
for ft in "implicit=4" "implicit=4,cluster=1" "implicit=2" "implicit=3" "implicit=3,cluster=1" "implicit=4,split=2" "implicit=4,split=3"; do
  echo "== $ft" >> $o
  timeout 200 python tools/time_one.py mcc_bf16 --reps 20 --force-tile $ft >> $o 2>&1
done
echo "== plain GEMM same MNK" >> $o
timeout 200 python tools/time_one.py mm:12544,512,4608 mm:4096,4096,4096 mm:8192,8192,8192 --reps 20 >> $o 2>&1
timeout 200 python tools/time_one.py mm:12544,512,4608 --reps 20 --force-tile cluster=1 >> $o 2>&1
timeout 200 python tools/time_one.py mm:12544,512,4608 mm:4096,4096,4096 --reps 20 --force-tile split=2 >> $o 2>&1
echo "== cublas" >> $o
timeout 200 python tools/cublas_ref.py 12544,512,4608 4096,4096,4096 8192,8192,8192 >> $o 2>&1
cat $o
timeout 200 python tools/cudnn_ref.py 256 >> $o 2>&1; tail -3 $o
