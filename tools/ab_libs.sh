# A/B the library variants given as paper_conf_sc_fallingsb23_b200/libeclmst_<name>.so on configs:
#   bash tools/ab_libs.sh <tag> "<names>" "<configs>"   (name "base" = the default build)
TAG=$1; NAMES=$2; CFGS=$3
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for c in $CFGS; do for v in $NAMES; do
  if [ "$v" = base ]; then L=$PWD/paper_conf_sc_fallingsb23_b200/libeclmst.so; else L=$PWD/paper_conf_sc_fallingsb23_b200/libeclmst_$v.so; fi
  ECLMST_LIB=$L timeout 300 python bench.py --config $c --parity none --no-e2e --no-cpu-baseline --steps 7 > gpurun_out/${TAG}_${v}_${c}.json 2>/dev/null
  python tools/bench_brief.py gpurun_out/${TAG}_${v}_${c}.json | sed "s|gpurun_out/||" | cut -c1-60,200-420
done; done
