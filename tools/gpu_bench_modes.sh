cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python bench.py --config road --dist --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bm_dist_road.json 2> gpurun_out/bm_dist_road.err; echo "dist road rc=$?"; tail -c 1500 gpurun_out/bm_dist_road.json; tail -3 gpurun_out/bm_dist_road.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bm_trun.json 2> gpurun_out/bm_trun.err; echo "torchrun rc=$?"; head -c 400 gpurun_out/bm_trun.json; echo
timeout 600 python bench.py --impl reference --steps 1 --warmup 0 > gpurun_out/bm_ref.json 2> gpurun_out/bm_ref.err; echo "ref rc=$?"; cat gpurun_out/bm_ref.json
