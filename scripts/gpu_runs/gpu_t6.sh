L=$PWD/paper_conf_sc_chenbpbyo22_b200
for n in default ku8 ku2 t1024; do
  if [ $n = default ]; then export ATOS_LIB=$L/libatos.so; else export ATOS_LIB=$L/libatos_$n.so; fi
  echo "== $n" >> gpurun_out/t6_exp.log
  timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"hub_cache":0}, {"hub_cache":0, "relabel":0}]' 2>&1 | grep cfg >> gpurun_out/t6_exp.log
  if [ $n = default ] || [ $n = ku8 ]; then
    timeout 600 python scripts/exp_pr.py --configs '[{}, {"relabel":0}]' 2>&1 | grep cfg >> gpurun_out/t6_exp.log
    timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{"hub_cache":0}]' 2>&1 | grep cfg >> gpurun_out/t6_exp.log
    timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{"hub_cache":0}]' 2>&1 | grep cfg >> gpurun_out/t6_exp.log
  fi
done
