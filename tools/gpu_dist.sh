# sharded-path check on one GPU: bash tools/gpu_dist.sh <tag> [configs...]
TAG=${1:-d}; shift; CFGS=${@:-road rmat}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_dist.py -m gpu -x -q > gpurun_out/pytest_dist_${TAG}.log 2>&1; echo "pytest dist rc=$?"; tail -3 gpurun_out/pytest_dist_${TAG}.log
for c in $CFGS; do
    timeout 900 python bench.py --dist --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bdist_${TAG}_${c}.json 2> gpurun_out/bdist_${TAG}_${c}.err
    echo "dist $c rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/bdist_${TAG}_${c}.json')); print(d['ms_per_step'], d.get('parity_vs_oracle'), d['stats']['rounds'])"
    tail -2 gpurun_out/bdist_${TAG}_${c}.err
done
