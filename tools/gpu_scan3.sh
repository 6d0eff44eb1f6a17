# T6: register row scan after the column fold, launched with programmatic stream serialization
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
o=gpurun_out/scan3.txt
: > $o
timeout 900 python -m pytest tests -q -m gpu -k "scan or ps or prefix or mbbs" >> $o 2>&1
for rep in 1 2 3; do
timeout 300 python tools/time_one.py mbbs_f32 prefix_sum_f32 --reps 20 2>&1 | cut -c1-110 >> $o
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/scan3_launches.csv python tools/profile_one.py --workload mbbs_f32 --reps 3 >> $o 2>&1
timeout 300 compute-sanitizer --tool memcheck python tools/profile_one.py --workload mbbs_f32 --reps 1 2>&1 | tail -3 >> $o
cat $o
