cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/caps.txt
: > $o
MDH_DEBUG_SYNC=1 timeout 400 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "caps or mcc or variants" >> $o 2>&1; echo "tests rc=$?" >> $o
timeout 200 python tools/time_one.py mcc_caps_bf16 --reps 10 2>&1 | cut -c1-160 >> $o
timeout 200 python tools/time_one.py mcc_caps_bf16 --reps 10 --force-tile implicit=3 2>&1 | cut -c1-160 >> $o
timeout 600 compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize_cases.py t4_ag4 >> $o 2>&1; echo "memcheck rc=$?" >> $o
tail -8 $o
