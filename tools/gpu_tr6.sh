cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 200 python tools/t4_trace.py mm:4096,4096,4096 --force-tile bn=512,split=2 > gpurun_out/trace_t6a.jsonl 2>&1
timeout 200 python tools/t4_trace.py mm:4096,4096,4096 --force-tile bn=512,split=1 > gpurun_out/trace_t6b.jsonl 2>&1
grep span gpurun_out/trace_t6*.jsonl | cut -c1-400
