# usage: bash tools/gpu_ncu.sh <tag> <config...> : one ncu --set full capture of the persistent kernel per config
TAG=$1; shift
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for CFG in "$@"; do
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:mst_persistent -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_${CFG} -f python tools/profile_run.py --config $CFG --runs 2 > gpurun_out/prof_${TAG}_${CFG}.log 2>&1
echo "$CFG ncu rc=$?"; tail -2 gpurun_out/prof_${TAG}_${CFG}.log
done
