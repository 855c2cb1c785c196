for rep in 1 2; do
for mode in dyn static; do
  unset ATOS_STATIC_CHUNKS
  if [ $mode = static ]; then export ATOS_STATIC_CHUNKS=1; fi
  echo "== $mode" >> gpurun_out/s4e.log
  timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep cfg >> gpurun_out/s4e.log
  timeout 300 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/s4e.log
  timeout 300 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0}]' 2>&1 | grep cfg >> gpurun_out/s4e.log
done
done
export ATOS_STATIC_CHUNKS=1
timeout 900 python -m pytest tests/test_gpu_bfs.py tests/test_gpu_pagerank.py -m gpu -x -q -p no:cacheprovider > gpurun_out/s4e_tests.log 2>&1; echo rc=$? >> gpurun_out/s4e_tests.log
