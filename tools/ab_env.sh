# A/B an environment setting on configs:  bash tools/ab_env.sh <tag> "<VAR=val ...>" "<configs>"   ("-" = unset)
TAG=$1; SETS=$2; CFGS=$3
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for c in $CFGS; do for kv in $SETS; do
  if [ "$kv" = "-" ]; then E=""; N=base; else E="$kv"; N=$(echo $kv | tr '=' '_'); fi
  env $E timeout 300 python bench.py --config $c --parity none --no-e2e --no-cpu-baseline --steps 7 > gpurun_out/${TAG}_${N}_${c}.json 2>/dev/null
  python tools/bench_brief.py gpurun_out/${TAG}_${N}_${c}.json | sed "s|gpurun_out/||" | cut -c1-60,200-420
done; done
