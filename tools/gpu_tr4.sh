cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/tr4.txt
: > $o
for ft in "bn=512" "bn=256" "bn=512,split=1"; do
timeout 200 python tools/time_one.py mcc_bf16 matmul_bf16 --reps 20 --force-tile $ft 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print('$ft', d['workload'], d['ms'], d['value'], d['frac'])
    except Exception: print(l.strip()[:200])" >> $o
done
timeout 200 python tools/t4_trace.py mcc_bf16 matmul_bf16 > gpurun_out/trace_t4.jsonl 2>&1
timeout 200 python tools/t4_trace.py mcc_bf16 --force-tile bn=256 > gpurun_out/trace_t4n.jsonl 2>&1
grep span gpurun_out/trace_t4*.jsonl | cut -c1-250 >> $o
cat $o
