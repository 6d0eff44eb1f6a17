cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/wide.txt
: > $o
MDH_DEBUG_SYNC=1 timeout 60 python tools/time_one.py mm:1024,1024,1024 --reps 2 --force-tile bn=512 >> $o 2>&1; echo "smoke rc=$?" >> $o
if grep -q '"ms"' $o; then
MDH_DEBUG_SYNC=1 timeout 400 python -m pytest tests/test_gpu_parity.py -q -m gpu -x --timeout=120 -k "stream_k or im2col" >> $o 2>&1; echo "tests rc=$?" >> $o
for ft in "bn=256" "bn=512"; do
timeout 200 python tools/time_one.py matmul_bf16 mcc_bf16 mm:12544,512,4608 mm:8192,8192,8192 --reps 20 --force-tile $ft >> $o 2>&1
done
timeout 200 python tools/t4_trace.py mm:4096,4096,4096 mm:12544,512,4608 mcc_bf16 --force-tile bn=512 > gpurun_out/trace_w.jsonl 2>&1
grep span gpurun_out/trace_w.jsonl >> $o
fi
tail -14 $o
