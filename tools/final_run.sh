TAG=${1:-r02g}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
bash tools/gpu_run.sh $TAG info tests slow bench:uniform
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_bench_reference.json 2> gpurun_out/${TAG}_bench_reference.err; echo "ref rc=$?"
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/${TAG}_smoke.log
bash tools/gpu_run.sh $TAG profile:uniform profile:road quick:road quick:rmat quick:rgg quick:grid
