for n in t256 ku16 ku4; do
  echo "== $n" >> gpurun_out/t5_exp.log
  ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_$n.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"hub_cache":0}, {"hub_cache":0, "pipeline":0}, {}]' >> gpurun_out/t5_exp.log 2>&1
done
