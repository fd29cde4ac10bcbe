# full GPU check + profiles for the given configs: bash tools/gpu_round.sh <tag> <cfg...>
TAG=$1; shift
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
bash tools/gpu_check.sh $TAG "$@"
for c in "$@"; do bash tools/gpu_profile.sh $TAG $c; done
