timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests12.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests12.log
python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' > gpurun_out/exp12.log 2>&1
python scripts/prof_worker.py --app pr >> gpurun_out/exp12.log 2>&1
