ATOS_SAME_DEVICE=1 timeout 600 python -m torch.distributed.run --standalone --nproc-per-node 2 bench.py --gpus 2 --workload bfs_rmat18 --steps 4 --warmup 3 --ctas-per-sm 1 --e2e-steps 1 > gpurun_out/b25_mp.json 2> gpurun_out/b25_mp.err; echo rc=$? >> gpurun_out/b25_mp.err
timeout 900 python bench.py --workload bfs_rmat26 --steps 8 --no-pr > gpurun_out/b25_r26.json 2> gpurun_out/b25_r26.err
timeout 900 python bench.py --workload bfs_grid4900 --steps 3 --no-pr --e2e-steps 1 > gpurun_out/b25_grid.json 2> gpurun_out/b25_grid.err
