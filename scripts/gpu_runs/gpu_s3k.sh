L=$PWD/paper_conf_sc_chenbpbyo22_b200
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"hub_cache":65536}, {"hub_cache":16384}, {"probe_filter":1}, {"probe_filter":1,"hub_cache":65536}]' > gpurun_out/s3k_rmat24.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{}, {"hub_cache":65536}]' > gpurun_out/s3k_rmat26.log 2>&1
ATOS_LIB=$L/libatos_ku8.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"probe_filter":1}]' > gpurun_out/s3k_ku8.log 2>&1
ATOS_LIB=$L/libatos_prof.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' > gpurun_out/s3k_prof24.log 2>&1
