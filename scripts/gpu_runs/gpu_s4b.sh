for rep in 1 2; do
for mode in base wf early both; do
  unset ATOS_EARLY ATOS_WARP_FLUSH
  case $mode in wf) export ATOS_WARP_FLUSH=1;; early) export ATOS_EARLY=1;; both) export ATOS_EARLY=1 ATOS_WARP_FLUSH=1;; esac
  echo "== $mode" >> gpurun_out/s4b.log
  timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep cfg >> gpurun_out/s4b.log
  timeout 300 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/s4b.log
done
done
