ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_prof.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' > gpurun_out/t15.log 2>&1
bash scripts/gpu_exp.sh t15 0 rmat24 '[{}, {"worker_mode":0}]' grid4900 '[{}]'
python scripts/exp_pr.py --configs '[{"relabel":0}, {"relabel":0, "worker_mode":0}]' >> gpurun_out/t15_exp.log 2>&1
