timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3j_tests.log 2>&1; echo rc=$? >> gpurun_out/s3j_tests.log
timeout 600 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0}, {"relabel":0,"discrete":1}, {"relabel":0,"virtual_ranks":8}, {"relabel":0,"virtual_ranks":8,"pr_combine":1}, {"relabel":0,"virtual_ranks":2}]' > gpurun_out/s3j_pr20.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"discrete":1}, {"virtual_ranks":8}, {"virtual_ranks":2}]' > gpurun_out/s3j_rmat24.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"discrete":1}, {"virtual_ranks":4}]' > gpurun_out/s3j_grid.log 2>&1
