# usage: bash tools/gpu_ring.sh -- parity of the default build, then A/B of the exp/ ring variants
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_ring.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ring.log
bash tools/gpu_ab.sh "road rmat rgg grid" -- exp/r0.so exp/r2.so exp/r3.so exp/r4.so
