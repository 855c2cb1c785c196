L=$PWD/paper_conf_sc_chenbpbyo22_b200
for rep in 1 2 3; do
for lib in libatos_head.so libatos.so; do
  echo "== $lib" >> gpurun_out/s4f.log
  ATOS_LIB=$L/$lib timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep cfg >> gpurun_out/s4f.log
  ATOS_LIB=$L/$lib timeout 300 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0}]' 2>&1 | grep cfg >> gpurun_out/s4f.log
done
done
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s4f_tests.log 2>&1; echo rc=$? >> gpurun_out/s4f_tests.log
