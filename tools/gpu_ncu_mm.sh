cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/ncu_mm.txt
: > $o
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm2 -s 2 -c 1 -o gpurun_out/mm_ours -f python tools/profile_one.py --workload matmul_bf16 --reps 4 >> $o 2>&1
timeout 600 ncu --set full --clock-control none -k regex:'nvjet|gemm|sm100|cutlass' -s 2 -c 1 -o gpurun_out/mm_cublas -f python tools/cublas_one.py 4096,4096,4096 >> $o 2>&1
for r in mm_ours mm_cublas; do
  ncu -i gpurun_out/$r.ncu-rep --page raw --csv > gpurun_out/$r.raw.csv 2>&1
  ncu -i gpurun_out/$r.ncu-rep --page details --csv > gpurun_out/$r.details.csv 2>&1
done
tail -3 $o
