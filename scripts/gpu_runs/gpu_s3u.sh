for c in 1000000 2 4 8 16 32 64; do
  echo "== chain $c" >> gpurun_out/s3u_grid.log
  ATOS_KEEP_CHAIN=$c timeout 300 python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"keep_items":256}]' 2>&1 | grep cfg >> gpurun_out/s3u_grid.log
done
