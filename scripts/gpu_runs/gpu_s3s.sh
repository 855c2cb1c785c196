timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3s_tests.log 2>&1; echo rc=$? >> gpurun_out/s3s_tests.log
timeout 600 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0,"virtual_ranks":8}, {"relabel":0,"virtual_ranks":2}]' > gpurun_out/s3s_pr20.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"virtual_ranks":8}, {"virtual_ranks":2}, {}]' > gpurun_out/s3s_rmat24.log 2>&1
