ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_prof.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' > gpurun_out/t13.log 2>&1
bash scripts/gpu_exp.sh t13 0 rmat24 '[{}, {"worker_mode":0}]' grid4900 '[{}]'
python scripts/exp_pr.py --configs '[{"relabel":0}]' >> gpurun_out/t13_exp.log 2>&1
