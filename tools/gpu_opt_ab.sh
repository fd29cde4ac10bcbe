# usage: bash tools/gpu_opt_ab.sh "<configs>" "<opt set 1>" "<opt set 2>" ...   (opt set: "k=v k=v" or "-")
CFGS=$1; shift
cd $GRAFT_REPO_ROOT
for c in $CFGS; do for os in "$@"; do
  args=""; [ "$os" != "-" ] && for kv in $os; do args="$args --opt $kv"; done
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-parity $args > /tmp/ab.json 2>/tmp/ab.err
  python -c "
import json
d=json.load(open('/tmp/ab.json')); r=d['roofline']; s=d['stats']
print('$c', '[$os]', 'ms=%.3f'%d['ms_per_step'], {k: round(v,3) for k,v in r['stage_ms'].items() if v > 0.02}, 'rounds', s['rounds'], 'live', s['live'][:24])
" || tail -3 /tmp/ab.err
done; done
