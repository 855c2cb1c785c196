timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider -k "not multiprocess" > gpurun_out/gpu_tests20.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests20.log
for r in 1 2; do python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"pipeline":1}, {"pipeline":1, "relax_red":1}, {"relax_red":1}]' 2>&1 | grep cfg >> gpurun_out/exp20.log; done
python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"pipeline":1}]' 2>&1 | grep cfg >> gpurun_out/exp20.log
