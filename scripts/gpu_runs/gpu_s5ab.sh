L=$PWD/paper_conf_sc_chenbpbyo22_b200
for rep in 1 2; do
for mode in head hybrid dyn; do
  unset ATOS_DYNAMIC_CHUNKS; lib=libatos.so
  case $mode in head) lib=libatos_head.so;; dyn) export ATOS_DYNAMIC_CHUNKS=1;; esac
  echo "== $mode" >> gpurun_out/s5ab.log
  ATOS_LIB=$L/$lib timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep cfg >> gpurun_out/s5ab.log
  ATOS_LIB=$L/$lib timeout 300 python scripts/exp_bfs.py --graph rmat26 --configs '[{}, {}]' 2>&1 | grep cfg >> gpurun_out/s5ab.log
  ATOS_LIB=$L/$lib timeout 300 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0}]' 2>&1 | grep cfg >> gpurun_out/s5ab.log
done
done
