# usage: bash tools/gpu_profile.sh <tag> [config]  -- bench + ncu launch list + ncu full of one MSF
TAG=${1:-r01}; CFG=${2:-road}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python bench.py --config $CFG > gpurun_out/bench_${TAG}_${CFG}.json 2> gpurun_out/bench_${TAG}_${CFG}.err; echo "bench rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_${CFG}.csv \
  python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-parity > gpurun_out/launches_${TAG}_${CFG}.log 2>&1
echo "launches rc=$?"
case $CFG in road|grid) NK=4;; *) NK=9;; esac   # our kernels per MSF (filtered: + flatten x2, giant, populate2, rounds2)
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_" -s $NK -c $NK \
  -o gpurun_out/prof_${TAG}_${CFG} -f python tools/profile_run.py --config $CFG --runs 2 > gpurun_out/prof_${TAG}_${CFG}.log 2>&1
echo "full rc=$?"; tail -2 gpurun_out/prof_${TAG}_${CFG}.log
