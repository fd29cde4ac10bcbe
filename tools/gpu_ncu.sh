# usage: bash tools/gpu_ncu.sh <tag> <kernel-regex> <config...> : ncu --set full of the matching kernels (2nd run)
TAG=$1; KRX=$2; shift; shift
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for CFG in "$@"; do
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"$KRX" -s 7 -c 7 \
  -o gpurun_out/prof_${TAG}_${CFG} -f python tools/profile_run.py --config $CFG --runs 2 > gpurun_out/prof_${TAG}_${CFG}.log 2>&1
echo "$CFG ncu rc=$?"; tail -2 gpurun_out/prof_${TAG}_${CFG}.log
done
