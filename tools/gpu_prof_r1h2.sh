# r1h: ncu --set full of this session's changed kernels (streaming scan, MBBS fold + register row scan, MCC N=1 GEMM + fold)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r1h
for spec in "prefix_sum_f32 t6_stream_scan prof_prefix" "mbbs_f32 t6_colfold prof_mbbs_fold" "mbbs_f32 t6_rowscan4 prof_mbbs_rowscan" "mcc_bf16_n1 t4_xfold prof_mcc_n1_fold" "mcc_bf16_n1 gemm_kernel prof_mcc_n1_gemm"; do
  set -- $spec
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$2 -s 1 -c 1 -f \
      -o gpurun_out/r1h/$3 python tools/profile_one.py --workload $1 --reps 2 > gpurun_out/r1h/$3.log 2>&1
done
ls gpurun_out/r1h
