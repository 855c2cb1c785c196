export ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_prof.so
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' > gpurun_out/t12.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' >> gpurun_out/t12.log 2>&1
