timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s4d_tests.log 2>&1; echo rc=$? >> gpurun_out/s4d_tests.log
for rep in 1 2; do
for mode in map nomap; do
  unset ATOS_NO_EDGE_MAP
  if [ $mode = nomap ]; then export ATOS_NO_EDGE_MAP=1; fi
  echo "== $mode" >> gpurun_out/s4d.log
  timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep cfg >> gpurun_out/s4d.log
  timeout 300 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/s4d.log
  timeout 300 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0}]' 2>&1 | grep cfg >> gpurun_out/s4d.log
  timeout 300 python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/s4d.log
done
done
