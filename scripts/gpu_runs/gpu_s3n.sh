L=$PWD/paper_conf_sc_chenbpbyo22_b200
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3n_tests.log 2>&1; echo rc=$? >> gpurun_out/s3n_tests.log
ATOS_LOAD_TRACE=1 timeout 600 python scripts/load_timing.py rmat24 > gpurun_out/s3n_load.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"probe_filter":0}]' > gpurun_out/s3n_rmat24.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' > gpurun_out/s3n_rmat26.log 2>&1
ATOS_LIB=$L/libatos_carve.so timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' > gpurun_out/s3n_carve26.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' > gpurun_out/s3n_grid.log 2>&1
