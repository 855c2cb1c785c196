for i in 1 2; do
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider --durations=8 > gpurun_out/s3v_tests$i.log 2>&1; echo rc=$? >> gpurun_out/s3v_tests$i.log
done
for i in 1 2 3 4 5; do timeout 300 python -m pytest tests/test_gpu_pagerank.py -m gpu -q -p no:cacheprovider -k "config1" >> gpurun_out/s3v_pr.log 2>&1; done
for c in 1000000 2 4 8 16 32 64; do
  echo "== chain $c" >> gpurun_out/s3u_grid.log
  ATOS_KEEP_CHAIN=$c timeout 300 python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"keep_items":256}]' 2>&1 | grep cfg >> gpurun_out/s3u_grid.log
done
