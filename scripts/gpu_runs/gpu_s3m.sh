L=$PWD/paper_conf_sc_chenbpbyo22_b200
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"pipeline":1}, {"pipeline":0}]' > gpurun_out/s3m_base24.log 2>&1
ATOS_LIB=$L/libatos_pipe3.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"pipeline":3}, {"pipeline":3, "probe_filter":1}]' > gpurun_out/s3m_p3_24.log 2>&1
ATOS_LIB=$L/libatos_pipe3k2.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"pipeline":3}, {}, {"pipeline":3, "probe_filter":1}]' > gpurun_out/s3m_p3k2_24.log 2>&1
ATOS_LIB=$L/libatos_pipe3.so timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{}, {"pipeline":3}]' > gpurun_out/s3m_p3_26.log 2>&1
ATOS_LIB=$L/libatos_pipe3k2.so timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{"pipeline":3}]' > gpurun_out/s3m_p3k2_26.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3m_tests.log 2>&1; echo rc=$? >> gpurun_out/s3m_tests.log
timeout 600 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0,"virtual_ranks":8}, {"relabel":0,"virtual_ranks":2}, {"relabel":0,"virtual_ranks":4}]' > gpurun_out/s3m_pr20.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"virtual_ranks":8}, {"virtual_ranks":2}, {"virtual_ranks":4}]' > gpurun_out/s3m_rmat24.log 2>&1
