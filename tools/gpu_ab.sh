# usage: bash tools/gpu_ab.sh <configs> -- <lib1> <lib2> ... : bench every exp library on every config
CFGS=$1; shift; shift
cd $GRAFT_REPO_ROOT
for lib in "$@"; do for c in $CFGS; do
  ECLMST_LIB=$lib timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-parity > /tmp/ab.json 2>/tmp/ab.err
  python -c "
import json
d=json.load(open('/tmp/ab.json')); r=d['roofline']
print('$lib', '$c', 'ms=%.3f'%d['ms_per_step'], {k: round(v,3) for k,v in r['stage_ms'].items() if v > 0.02})
" || tail -3 /tmp/ab.err
done; done
