cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/cl4.txt
: > $o
MDH_DEBUG_SYNC=1 timeout 60 python tools/time_one.py mm:1024,1024,1024 --reps 2 >> $o 2>&1; echo "smoke rc=$?" >> $o
if grep -q '"ms"' $o; then
MDH_DEBUG_SYNC=1 timeout 300 python -m pytest tests/test_gpu_parity.py -q -m gpu -x --timeout=120 -k "stream_k" >> $o 2>&1; echo "sk tests rc=$?" >> $o
timeout 400 python -m pytest tests/test_gpu_parity.py -q -m gpu -x --timeout=120 -k "tcgen05 or mcc or matmul or t4" >> $o 2>&1; echo "t4 tests rc=$?" >> $o
timeout 200 python tools/time_one.py matmul_bf16 mcc_bf16 mm:12544,512,4608 mm:8192,8192,8192 --reps 20 >> $o 2>&1
timeout 200 python tools/time_one.py matmul_bf16 mcc_bf16 mm:12544,512,4608 mm:8192,8192,8192 --reps 20 --force-tile cluster=2 >> $o 2>&1
timeout 200 python tools/cublas_ref.py 4096,4096,4096 8192,8192,8192 >> $o 2>&1
timeout 200 python tools/t4_trace.py mm:4096,4096,4096 mm:12544,512,4608 mcc_bf16 > gpurun_out/trace_cl4.jsonl 2>gpurun_out/trace_cl4.err; cat gpurun_out/trace_cl4.err >> $o
grep span gpurun_out/trace_cl4.jsonl >> $o
fi
tail -14 $o
