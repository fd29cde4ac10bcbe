# usage: bash tools/gpu_opt_ab.sh "<configs>" "<opt sets separated by ;>"   e.g. "road rmat" "node_layout=1;node_layout=2"
CFGS=$1; OPTS=$2
cd $GRAFT_REPO_ROOT
IFS=';' read -ra SETS <<< "$OPTS"
for c in $CFGS; do for o in "${SETS[@]}"; do
  args=""; for kv in $o; do args="$args --opt $kv"; done
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-parity $args > /tmp/ab.json 2>/tmp/ab.err
  python -c "
import json
d=json.load(open('/tmp/ab.json')); r=d['roofline']
print('$c', '[$o]', 'ms=%.3f'%d['ms_per_step'], {k: round(v,3) for k,v in r['stage_ms'].items() if v > 0.02})
" || tail -3 /tmp/ab.err
done; done
