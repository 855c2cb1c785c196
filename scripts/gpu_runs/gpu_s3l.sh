timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3l_tests.log 2>&1; echo rc=$? >> gpurun_out/s3l_tests.log
timeout 600 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0,"virtual_ranks":8}, {"relabel":0,"virtual_ranks":2}, {"relabel":0,"virtual_ranks":8,"agg_batch_msgs":1024}]' > gpurun_out/s3l_pr20.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"virtual_ranks":8}, {"virtual_ranks":2}]' > gpurun_out/s3l_rmat24.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{"discrete":1}, {"virtual_ranks":4}, {"virtual_ranks":4,"keep_items":128,"keep_mode":1}]' > gpurun_out/s3l_grid.log 2>&1
L=$PWD/paper_conf_sc_chenbpbyo22_b200
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"hub_cache":65536}, {"hub_cache":16384}, {"probe_filter":1}, {"probe_filter":1,"hub_cache":65536}]' > gpurun_out/s3k_rmat24.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{}, {"hub_cache":65536}]' > gpurun_out/s3k_rmat26.log 2>&1
ATOS_LIB=$L/libatos_ku8.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"probe_filter":1}]' > gpurun_out/s3k_ku8.log 2>&1
ATOS_LIB=$L/libatos_prof.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' > gpurun_out/s3k_prof24.log 2>&1
