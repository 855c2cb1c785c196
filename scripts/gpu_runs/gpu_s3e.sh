# parity (split + combining), PR combining timings, grid keep sweep
L=$PWD/paper_conf_sc_chenbpbyo22_b200
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3e_tests.log 2>&1; echo rc=$? >> gpurun_out/s3e_tests.log
timeout 600 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0}, {"relabel":0,"virtual_ranks":8}, {"relabel":0,"virtual_ranks":8,"pr_combine":1}, {"relabel":0,"virtual_ranks":2,"pr_combine":1}, {"relabel":0,"virtual_ranks":2}]' > gpurun_out/s3e_pr20.log 2>&1
timeout 900 python scripts/exp_pr.py --graph rmat26_pr --reps 1 --configs '[{"relabel":0,"virtual_ranks":8,"pr_combine":1}]' > gpurun_out/s3e_pr26.log 2>&1
ATOS_LIB=$L/libatos_keepall.so timeout 900 python scripts/exp_bfs.py --graph grid4900 --configs '[{"relax_red":0,"keep_items":16}, {"relax_red":0,"keep_items":32}, {"relax_red":1,"keep_items":32}, {"relax_red":1,"keep_items":64}, {"relax_red":1,"keep_items":128}, {"relax_red":1,"keep_items":256}]' > gpurun_out/s3e_grid_keepall.log 2>&1
ATOS_LIB=$L/libatos_keepall.so timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"keep_items":0}, {"keep_items":64}]' > gpurun_out/s3e_rmat_keepall.log 2>&1
