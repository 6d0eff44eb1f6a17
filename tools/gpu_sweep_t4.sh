cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
cp tiles/b200.json gpurun_out/b200_before.json
timeout 900 python tools/sweep_tiles.py --only t4_ --reps 20 --out gpurun_out/b200.json > gpurun_out/sweep_t4.log 2>&1
cp gpurun_out/b200_before.json /dev/null
tail -20 gpurun_out/sweep_t4.log | cut -c1-150
