# A/B ecl_mst_options settings on configs:  bash tools/ab_opts.sh <tag> "<opt=val,opt=val ...>" "<configs>"   ("-" = defaults)
TAG=$1; SETS=$2; CFGS=$3
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for c in $CFGS; do for kv in $SETS; do
  if [ "$kv" = "-" ]; then A=""; N=base; else A=$(echo $kv | tr ',' '\n' | sed 's/^/--opt /' | tr '\n' ' '); N=$(echo $kv | tr '=,' '__'); fi
  timeout 300 python bench.py --config $c --parity none --no-e2e --no-cpu-baseline --steps 9 $A > gpurun_out/${TAG}_${N}_${c}.json 2>/dev/null
  python tools/bench_brief.py gpurun_out/${TAG}_${N}_${c}.json | sed "s|gpurun_out/||" | cut -c1-70,200-420
done; done
