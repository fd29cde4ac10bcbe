cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_dist.py -x -q > gpurun_out/pytest_dist.log 2>&1; echo "pytest dist rc=$?"; tail -3 gpurun_out/pytest_dist.log
timeout 600 python bench.py --config road --dist --steps 5 --no-cpu-baseline --no-parity --no-e2e > gpurun_out/bench_dist_road.json 2>gpurun_out/bench_dist_road.err; echo "dist bench rc=$?"; python -c "import json; d=json.load(open('gpurun_out/bench_dist_road.json')); print('dist road ms', d['ms_per_step'])"
timeout 600 python bench.py --config rmat --dist --steps 5 --no-cpu-baseline --no-parity --no-e2e > gpurun_out/bench_dist_rmat.json 2>gpurun_out/bench_dist_rmat.err; python -c "import json; d=json.load(open('gpurun_out/bench_dist_rmat.json')); print('dist rmat ms', d['ms_per_step'])"
timeout 1500 python tools/ablation.py --configs road rgg rmat grid --out gpurun_out/ablation_r01.json 2>&1 | tail -70
timeout 900 python tools/ablation.py --seeds 99 --runs 1 --configs rgg rmat --out gpurun_out/seeds_r01.json 2>&1 | tail -3
