L=$PWD/paper_conf_sc_chenbpbyo22_b200
for n in default w128; do
  if [ $n = default ]; then export ATOS_LIB=$L/libatos.so; else export ATOS_LIB=$L/libatos_$n.so; fi
  echo "== $n" >> gpurun_out/t16_exp.log
  timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"ctas_per_sm":2}]' 2>&1 | grep cfg >> gpurun_out/t16_exp.log
  timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/t16_exp.log
  timeout 600 python scripts/exp_pr.py --configs '[{"relabel":0}]' 2>&1 | grep cfg >> gpurun_out/t16_exp.log
done
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/t16_tests.log 2>&1; echo rc=$? >> gpurun_out/t16_tests.log
