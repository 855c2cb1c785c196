# row splitting: parity + sweep; grid; PR virtual-rank aggregation at RMAT-26
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3c_tests.log 2>&1; echo rc=$? >> gpurun_out/s3c_tests.log
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"split_edges":0},{"split_edges":-1},{"split_edges":1024},{"split_edges":2048},{"split_edges":8192}]' > gpurun_out/s3c_exp24.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{"split_edges":0},{"split_edges":-1},{"split_edges":2048}]' > gpurun_out/s3c_exp26.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"keep_items":64}, {"pipeline":0}]' > gpurun_out/s3c_grid.log 2>&1
timeout 900 python scripts/exp_pr.py --graph rmat26_pr --reps 1 --configs '[{"relabel":0}, {"relabel":0,"virtual_ranks":8,"agg_enabled":1}, {"relabel":0,"virtual_ranks":8,"agg_enabled":0}]' > gpurun_out/s3c_pr26.log 2>&1
