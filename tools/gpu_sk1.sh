cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/sk1.txt
: > $o
MDH_DEBUG_SYNC=1 timeout 300 python -m pytest tests/test_gpu_parity.py -q -m gpu -x --timeout=120 -k "stream_k" >> $o 2>&1; echo "sk tests rc=$?" >> $o
timeout 400 python -m pytest tests/test_gpu_parity.py -q -m gpu -x --timeout=120 -k "tcgen05 or mcc or matmul or t4" >> $o 2>&1; echo "t4 tests rc=$?" >> $o
timeout 200 python tools/time_one.py matmul_bf16 mcc_bf16 mm:12544,512,4608 mm:8192,8192,8192 --reps 20 >> $o 2>&1
timeout 200 python tools/time_one.py matmul_bf16 mcc_bf16 mm:12544,512,4608 --reps 20 --force-tile split=1 >> $o 2>&1
timeout 200 python tools/t4_trace.py mm:4096,4096,4096 mm:12544,512,4608 mcc_bf16 > gpurun_out/trace_sk.jsonl 2>&1
grep span gpurun_out/trace_sk.jsonl >> $o
tail -12 $o
