timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests14.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests14.log
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"prefetch":0}, {}, {"prefetch":0}]' > gpurun_out/exp14.log 2>&1
python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' >> gpurun_out/exp14.log 2>&1
