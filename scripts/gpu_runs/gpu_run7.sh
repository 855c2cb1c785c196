timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests7.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests7.log
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"l2_persist":0}]' > gpurun_out/exp7.log 2>&1
python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' >> gpurun_out/exp7.log 2>&1
