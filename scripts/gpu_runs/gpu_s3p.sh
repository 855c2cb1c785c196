timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3p_tests.log 2>&1; echo rc=$? >> gpurun_out/s3p_tests.log
for e in 0 1; do
  if [ $e = 1 ]; then export ATOS_NO_EARLY=1; fi
  echo "== no_early=$e" >> gpurun_out/s3p_exp.log
  timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep cfg >> gpurun_out/s3p_exp.log
  timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/s3p_exp.log
  timeout 600 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0}]' 2>&1 | grep cfg >> gpurun_out/s3p_exp.log
  timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/s3p_exp.log
done
