python scripts/exp_pr.py --configs '[{}, {"l2_persist":0}, {"prefetch":0}]' > gpurun_out/exp21.log 2>&1
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"l2_persist":0}]' 2>&1 | grep cfg >> gpurun_out/exp21.log
