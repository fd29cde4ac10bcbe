# per-kernel launch list of one sharded MSF (ncu, serialised) + A/B of refilter on the sharded path
TAG=${1:-dp}; CFG=${2:-road}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for o in "refilter=0" "refilter=-1"; do
  timeout 600 python bench.py --dist --config $CFG --steps 7 --warmup 3 --no-cpu-baseline --no-e2e --no-parity --opt $o > /tmp/d.json 2>/dev/null
  python -c "
import json; d=json.load(open('/tmp/d.json')); print('$CFG $o', d['ms_per_step'], d['stats']['rounds'], d['stats'].get('refilters'), d['stats']['live'][:20])"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/dlaunch_${TAG}_${CFG}.csv \
  python bench.py --dist --config $CFG --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-parity > /dev/null 2>&1
echo "ncu rc=$?"
