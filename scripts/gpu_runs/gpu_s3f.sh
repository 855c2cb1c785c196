timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3f_tests.log 2>&1; echo rc=$? >> gpurun_out/s3f_tests.log
timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"keep_items":0}]' > gpurun_out/s3f_grid.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"probe_filter":1}, {"probe_filter":1, "l2_persist":0}]' > gpurun_out/s3f_rmat24.log 2>&1
timeout 600 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0,"virtual_ranks":8}, {"relabel":0,"virtual_ranks":8,"pr_combine":1}, {"relabel":0,"virtual_ranks":2}, {"relabel":0,"virtual_ranks":2,"pr_combine":1}, {"relabel":0,"virtual_ranks":8,"agg_batch_msgs":1024}]' > gpurun_out/s3f_pr20.log 2>&1
timeout 900 python scripts/exp_pr.py --graph rmat26_pr --reps 1 --configs '[{"relabel":0,"virtual_ranks":8}, {"relabel":0,"virtual_ranks":8,"pr_combine":1}]' > gpurun_out/s3f_pr26.log 2>&1
