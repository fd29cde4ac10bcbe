# usage: bash tools/gpu_profile.sh <tag> [config]
TAG=${1:-r01}; CFG=${2:-road}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python tools/profile_run.py --config $CFG --runs 2 > gpurun_out/prof_${TAG}_plain.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv \
  python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-parity > gpurun_out/launches_${TAG}.bench.log 2>&1
echo "launches rc=$?"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:mst_persistent -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_${CFG} -f python tools/profile_run.py --config $CFG --runs 2 > gpurun_out/prof_${TAG}.log 2>&1
echo "full rc=$?"
tail -3 gpurun_out/prof_${TAG}.log
