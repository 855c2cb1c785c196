timeout 900 python -m pytest tests -m gpu -x -q --timeout 120 -p no:cacheprovider > gpurun_out/gpu_tests16.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests16.log
timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"relax_red":1}, {}, {"relax_red":1}]' > gpurun_out/exp16.log 2>&1
timeout 300 python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' >> gpurun_out/exp16.log 2>&1
timeout 300 python scripts/prof_worker.py --app pr >> gpurun_out/exp16.log 2>&1
