timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests3.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests3.log
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"keep_items":0}, {"fetch_size":256}]' > gpurun_out/exp3.log 2>&1
python scripts/exp_bfs.py --graph path1000000 --configs '[{}]' >> gpurun_out/exp3.log 2>&1
python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"keep_items":0}, {"keep_items":256}]' >> gpurun_out/exp3.log 2>&1
