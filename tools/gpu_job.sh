#!/bin/bash
# One gpurun call's work, as a list of steps; every output lands in gpurun_out/<TAG>/.
#
#   gpurun --timeout 1200 -- 'bash tools/gpu_job.sh <TAG> <STEP> [<STEP> ...]'
#
# steps (each bounded by its own timeout so a hang cannot eat the call):
#   test[:<pytest -k expr>]           pytest -m gpu (all, or the -k selection)          -> tests.log
#   time:<w1+w2+..>[@<force_tile>]    tools/time_one.py device timings (L2 flushed)     -> time.jsonl
#   ncu:<kernel regex>:<workload>     ncu --set full of one launch of the kernel        -> ncu_<workload>.ncu-rep
#   launches[:<bench args>]           ncu launch list of a short bench run              -> launches.csv
#   bench[:<bench args>]              python bench.py (default args)                    -> bench.json
#   ref                               python bench.py --impl reference                  -> ref.json
#   smoke                             __graft_entry__.smoke()                           -> smoke.log
#   sweep:<args>                      tools/sweep_tiles.py (table copy updated)         -> sweep.log, b200.json
#   py:<script args>                  python <script args>                              -> py.log
#   torchrun:<N>:<bench args>         torchrun --nproc-per-node N bench.py ...          -> torchrun.log
set -u
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
TAG=$1
shift
OUT=gpurun_out/$TAG
mkdir -p "$OUT"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > "$OUT/gpu.txt" 2>&1
for step in "$@"; do
  kind=${step%%:*}
  arg=${step#*:}
  [ "$arg" = "$step" ] && arg=""
  echo "== $step" >> "$OUT/steps.log"
  case $kind in
    test)
      if [ -n "$arg" ]; then timeout 1500 python -m pytest tests -q -m gpu -k "$arg" >> "$OUT/tests.log" 2>&1
      else timeout 1500 python -m pytest tests -q -m gpu >> "$OUT/tests.log" 2>&1; fi
      echo "tests rc=$?" >> "$OUT/tests.log"; tail -3 "$OUT/tests.log" ;;
    time)
      wl=${arg%%@*}; ft=""
      [ "$wl" != "$arg" ] && ft="--force-tile ${arg#*@}"
      timeout 900 python tools/time_one.py ${wl//+/ } --reps 10 $ft >> "$OUT/time.jsonl" 2>> "$OUT/time.err"
      tail -5 "$OUT/time.jsonl" ;;
    ncu)
      k=${arg%%:*}; wl=${arg#*:}
      timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$k" -s 1 -c 1 -f \
        -o "$OUT/ncu_$wl" python tools/profile_one.py --workload "$wl" --reps 2 > "$OUT/ncu_$wl.log" 2>&1
      echo "ncu $wl rc=$?" ;;
    launches)
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
        --log-file "$OUT/launches.csv" python bench.py --steps 2 --warmup 3 ${arg:---no-suite --no-cpu-baseline} \
        > "$OUT/launches.log" 2>&1
      echo "launches rc=$?" ;;
    bench)
      timeout 1200 python bench.py $arg > "$OUT/bench.json" 2> "$OUT/bench.err"; echo "bench rc=$?"; tail -c 600 "$OUT/bench.json" ;;
    ref)
      timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > "$OUT/ref.json" 2> "$OUT/ref.err"; echo "ref rc=$?" ;;
    smoke)
      timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > "$OUT/smoke.log" 2>&1
      tail -2 "$OUT/smoke.log" ;;
    sweep)
      cp tiles/b200.json "$OUT/b200.json"     # the updated table comes back in gpurun_out/
      timeout 2400 python tools/sweep_tiles.py --out "$OUT/b200.json" $arg > "$OUT/sweep.log" 2>&1; echo "sweep rc=$?"; tail -5 "$OUT/sweep.log" ;;
    py)
      timeout 1200 python $arg >> "$OUT/py.log" 2>&1; echo "py rc=$?"; tail -15 "$OUT/py.log" ;;
    torchrun)
      n=${arg%%:*}; ba=${arg#*:}
      timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node "$n" --master-addr 127.0.0.1 \
        --master-port 29511 bench.py --gpus "$n" $ba >> "$OUT/torchrun.log" 2>&1
      echo "torchrun rc=$?"; tail -5 "$OUT/torchrun.log" ;;
    *)
      echo "unknown step $step" ;;
  esac
done
