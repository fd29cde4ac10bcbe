# GPU-box driver for gpurun:  bash tools/gpu_run.sh <tag> <step...>
#   info                 host cores / memory, GPU
#   tests                pytest -m "gpu and not slow"
#   slow                 pytest -m "gpu and slow" (full-size C3/C4/C5 vs the oracle, ids > 2^31)
#   bench:<cfg>          bench.py --config <cfg> (full oracle parity)
#   quick:<cfg>          bench.py --config <cfg> --parity none --no-e2e --no-cpu-baseline
#   profile:<cfg>        ncu launch list of the bench command + ncu --set full of one MSF
# Outputs land in gpurun_out/<tag>_*.
TAG=$1; shift
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for STEP in "$@"; do
  CFG=${STEP#*:}
  case $STEP in
    info) (nproc; free -g; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv) > gpurun_out/${TAG}_info.txt 2>&1
          cat gpurun_out/${TAG}_info.txt;;
    tests) timeout 900 python -m pytest tests -q -x -m "gpu and not slow" > gpurun_out/${TAG}_pytest.txt 2>&1
           echo "tests rc=$?"; tail -3 gpurun_out/${TAG}_pytest.txt;;
    slow) timeout 3000 python -m pytest tests -q -x -m "gpu and slow" --durations=10 > gpurun_out/${TAG}_pytest_slow.txt 2>&1
          echo "slow rc=$?"; tail -15 gpurun_out/${TAG}_pytest_slow.txt;;
    bench:*) T0=$SECONDS; timeout 1700 python bench.py --config $CFG > gpurun_out/${TAG}_bench_${CFG}.json 2> gpurun_out/${TAG}_bench_${CFG}.err
             echo "bench $CFG rc=$? wall=$((SECONDS-T0))s"; tail -3 gpurun_out/${TAG}_bench_${CFG}.err
             python tools/bench_brief.py gpurun_out/${TAG}_bench_${CFG}.json;;
    quick:*) timeout 300 python bench.py --config $CFG --parity none --no-e2e --no-cpu-baseline $QUICK_ARGS > gpurun_out/${TAG}_quick_${CFG}.json 2> gpurun_out/${TAG}_quick_${CFG}.err
             echo "quick $CFG rc=$?"; python tools/bench_brief.py gpurun_out/${TAG}_quick_${CFG}.json;;
    profile:*)
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_${CFG}.csv \
        python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --parity none > gpurun_out/${TAG}_launches_${CFG}.log 2>&1
      echo "launches rc=$?"
      case $CFG in road|grid) NK=4;; *) NK=10;; esac
      timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_" -s $NK -c $NK \
        -o gpurun_out/${TAG}_prof_${CFG} -f python tools/profile_run.py --config $CFG --runs 2 > gpurun_out/${TAG}_prof_${CFG}.log 2>&1
      echo "full rc=$?"; tail -2 gpurun_out/${TAG}_prof_${CFG}.log;;
  esac
done
