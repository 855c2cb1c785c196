ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_prof.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"prefetch":0}]' > gpurun_out/t14.log 2>&1
bash scripts/gpu_exp.sh t14 0 rmat24 '[{"prefetch":0}, {"worker_mode":0, "prefetch":0}]' grid4900 '[{"prefetch":0}]'
