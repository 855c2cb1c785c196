timeout 1200 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider -k "not multiprocess" > gpurun_out/gpu_tests26.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests26.log
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"probe_filter":1}]' 2>&1 | grep cfg >> gpurun_out/exp26.log
python scripts/exp_bfs.py --graph rmat26 --configs '[{}, {"probe_filter":0}]' 2>&1 | grep cfg >> gpurun_out/exp26.log
