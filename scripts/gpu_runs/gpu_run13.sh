timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests13.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests13.log
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"prefetch":0}, {}, {"prefetch":0}]' > gpurun_out/exp13.log 2>&1
