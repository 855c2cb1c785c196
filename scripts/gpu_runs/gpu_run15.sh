timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests15.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests15.log
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"relax_red":1}, {}, {"relax_red":1}]' > gpurun_out/exp15.log 2>&1
python scripts/exp_bfs.py --graph grid4900 --configs '[{"relax_red":1}]' >> gpurun_out/exp15.log 2>&1
