# end-of-round evidence after the sharded-path work: full pytest -m gpu, single-GPU bench+ncu for road/rmat,
# bench for grid/rgg/uniform, sharded x1 bench for all five
TAG=${1:-r01i}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
bash tools/gpu_round.sh $TAG road rmat
for c in grid rgg uniform; do
  timeout 900 python bench.py --config $c > gpurun_out/bench_${TAG}_${c}.json 2> gpurun_out/bench_${TAG}_${c}.err; echo "bench $c rc=$?"
  python -c "
import json; d=json.load(open('gpurun_out/bench_${TAG}_${c}.json')); print('$c', d['ms_per_step'], d['roofline']['stage'], d['roofline']['frac'], d.get('parity_vs_oracle'))"
done
for c in grid road rgg rmat uniform; do
  timeout 900 python bench.py --dist --config $c --no-cpu-baseline > gpurun_out/bdist_${TAG}_${c}.json 2> gpurun_out/bdist_${TAG}_${c}.err; echo "dist $c rc=$?"
  python -c "
import json; d=json.load(open('gpurun_out/bdist_${TAG}_${c}.json')); print('dist $c', d['ms_per_step'], d.get('parity_vs_oracle'), d['e2e']['ms_per_step'] if d.get('e2e') else None)"
done
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_${TAG}.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke_${TAG}.log
