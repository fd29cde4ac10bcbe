# usage: bash tools/gpu_opt_ab2.sh "<configs>" "<opt sets, ';'-separated, 'none' = defaults>" [reps]
CFGS=$1; OPTS=$2; REPS=${3:-1}
cd $GRAFT_REPO_ROOT
IFS=';' read -ra SETS <<< "$OPTS"
for r in $(seq $REPS); do for c in $CFGS; do for os in "${SETS[@]}"; do
  args=""; [ "$os" != none ] && for kv in $os; do args="$args --opt $kv"; done
  timeout 600 python bench.py --config $c --steps 7 --warmup 3 --no-e2e --no-cpu-baseline $args > /tmp/ab.json 2>/tmp/ab.err
  python -c "
import json
d=json.load(open('/tmp/ab.json')); r=d['roofline']
print('$c', '[$os]', 'ms=%.3f'%d['ms_per_step'], 'parity=%s'%d.get('parity_vs_oracle'), {k: round(v,3) for k,v in r['stage_ms'].items() if v > 0.02})
" || tail -3 /tmp/ab.err
done; done; done
