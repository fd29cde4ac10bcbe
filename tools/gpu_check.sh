# usage: bash tools/gpu_check.sh <tag> [bench configs...]
TAG=${1:-x}; shift
CFGS=${@:-road}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_${TAG}.log 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_gpu_${TAG}.log
for c in $CFGS; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/bench_${TAG}_${c}.json 2> gpurun_out/bench_${TAG}_${c}.err; echo "bench $c rc=$?"
  python -c "
import json,sys
d=json.load(open('gpurun_out/bench_${TAG}_${c}.json'))
print('$c', 'ms=%.3f'%d['ms_per_step'], 'Gedges/s=%.2f'%(d['value']/1e9), 'frac=%.3f'%d['roofline']['frac'], 'parity=',d['parity_vs_oracle'], 'rounds=',d['stats']['rounds'], d['stats']['stage_us'])
" 2>&1 | tail -2
  tail -3 gpurun_out/bench_${TAG}_${c}.err
done
