cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 200 python tools/t4_trace.py mm:12544,512,4608 mcc_bf16 > gpurun_out/trace_w3.jsonl 2>&1
grep span gpurun_out/trace_w3.jsonl | cut -c1-200
