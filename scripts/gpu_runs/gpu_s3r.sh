L=$PWD/paper_conf_sc_chenbpbyo22_b200
ATOS_LIB=$L/libatos_minb3.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"ctas_per_sm":3}, {"ctas_per_sm":2}]' > gpurun_out/s3r_minb3.log 2>&1
ATOS_LIB=$L/libatos_t256.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"ctas_per_sm":6}, {"ctas_per_sm":4}]' > gpurun_out/s3r_t256.log 2>&1
ATOS_LIB=$L/libatos_minb3.so timeout 600 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0,"ctas_per_sm":3}]' > gpurun_out/s3r_minb3_pr.log 2>&1
