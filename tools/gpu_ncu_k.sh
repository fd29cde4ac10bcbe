# usage: bash tools/gpu_ncu_k.sh <tag> <config> <kernel-regex> <skip> <count>
TAG=$1; CFG=$2; KRX=$3; SKIP=${4:-0}; CNT=${5:-1}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"$KRX" -s $SKIP -c $CNT \
  -o gpurun_out/prof_${TAG}_${CFG} -f python tools/profile_run.py --config $CFG --runs 2 > gpurun_out/prof_${TAG}_${CFG}.log 2>&1
echo "ncu rc=$?"; tail -2 gpurun_out/prof_${TAG}_${CFG}.log
