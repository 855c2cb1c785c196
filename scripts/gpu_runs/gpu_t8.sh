ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_prof.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' > gpurun_out/t8_prof.log 2>&1
ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_prof.so timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' >> gpurun_out/t8_prof.log 2>&1
bash scripts/gpu_prof.sh ku4 bfs rmat24 '{}'
