# usage: bash tools/gpu_ab_parity.sh "<configs>" lib1 lib2 ... -- GPU parity of the default build, then A/B
CFGS=$1; shift
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_ab.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab.log
bash tools/gpu_ab.sh "$CFGS" -- "$@"
