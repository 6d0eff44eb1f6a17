cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/trace1.txt
: > $o

timeout 200 python tools/t4_trace.py mm:4096,4096,4096 mm:12544,512,4608 mcc_bf16 > gpurun_out/trace_a.jsonl 2>&1
timeout 200 python tools/t4_trace.py mm:4096,4096,4096 mm:12544,512,4608 mcc_bf16 --force-tile split=2 > gpurun_out/trace_b.jsonl 2>&1
timeout 200 python tools/t4_trace.py mm:8192,8192,8192 > gpurun_out/trace_c.jsonl 2>&1
grep span gpurun_out/trace_*.jsonl >> $o
tail -5 $o
