./scripts/micro > gpurun_out/micro.json 2>&1
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"probe_filter":1}, {"probe_filter":1, "l2_persist":0}, {"l2_persist":0}]' > gpurun_out/exp8.log 2>&1
