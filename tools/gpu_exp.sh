# usage: bash tools/gpu_exp.sh <tag>   -- experiment batch (edit freely)
TAG=$1
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_${TAG}.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_${TAG}.log
for c in rmat road; do
  timeout 300 python tools/trace_run.py --config $c 2>&1 | tail -40
done
timeout 300 python tools/trace_run.py --config rmat --opt atomic_guards=0 2>&1 | head -3
timeout 300 python tools/trace_run.py --config road --opt atomic_guards=0 2>&1 | head -3
timeout 300 python tools/trace_run.py --config rgg 2>&1 | head -3
timeout 300 python tools/trace_run.py --config rgg --opt atomic_guards=0 2>&1 | head -3
