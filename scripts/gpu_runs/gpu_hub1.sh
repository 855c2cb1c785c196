# hub cache + relabel: GPU tests, then BFS configs on RMAT-24 / RMAT-26
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/hub1_tests.log 2>&1; echo rc=$? >> gpurun_out/hub1_tests.log
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"relabel":1,"hub_cache":0}, {"relabel":0}, {"relabel":1,"hub_cache":65536}]' > gpurun_out/hub1_exp.log 2>&1
python scripts/exp_bfs.py --graph rmat26 --configs '[{}, {"relabel":1,"hub_cache":0}, {"relabel":0}]' >> gpurun_out/hub1_exp.log 2>&1
