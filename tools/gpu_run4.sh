cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q -rf --timeout 600 > gpurun_out/run4_tests.txt 2>&1
timeout 900 python bench.py > gpurun_out/run4_bench.json 2> gpurun_out/run4_bench.err
MDH_BENCH_BACKEND=gloo MDH_BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29555 bench.py --gpus 2 --steps 5 --warmup 3 > gpurun_out/run4_n2.json 2> gpurun_out/run4_n2.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/run4_ref.json 2> gpurun_out/run4_ref.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/run4_smoke.txt 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r1_launches_bench.csv python bench.py --steps 2 --warmup 3 --no-suite --no-cpu-baseline > /dev/null 2>&1
for w in matmul_bf16 matmul_f32 jacobi3d ccsd_bf16 mcc_bf16 dot_f32 prefix_sum_f32 mbbs_f32; do
  timeout 600 ncu --set full --clock-control none --import-source on -s 2 -c 3 -o gpurun_out/prof2_$w python tools/profile_one.py --workload $w --reps 2 > gpurun_out/prof2_$w.log 2>&1
done
echo done
