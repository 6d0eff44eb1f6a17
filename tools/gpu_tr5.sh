cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 200 python tools/t4_trace.py mcc_bf16 matmul_bf16 > gpurun_out/trace_t5.jsonl 2>&1
grep span gpurun_out/trace_t5.jsonl | cut -c1-300
