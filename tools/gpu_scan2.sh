# T6 streaming scan: whole K-runs loaded into registers before the sequential adds
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/scan2.txt
: > $o
for rep in 1 2 3; do
timeout 300 python tools/time_one.py prefix_sum_f32 mbbs_f32 --reps 20 2>&1 | cut -c1-110 >> $o
done
timeout 900 python -m pytest tests -q -m gpu -k "scan or ps or prefix or mbbs" >> $o 2>&1
cat $o
