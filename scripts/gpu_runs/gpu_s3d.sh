# split sweep (noise check), grid latency variants
L=$PWD/paper_conf_sc_chenbpbyo22_b200
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"split_edges":512},{"split_edges":1024},{"split_edges":2048},{"split_edges":0},{"split_edges":1024},{"split_edges":2048}]' > gpurun_out/s3d_exp24.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{"split_edges":1024},{"split_edges":2048},{"split_edges":4096}]' > gpurun_out/s3d_exp26.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{"relax_red":0}, {"relax_red":0,"pipeline":0}, {"relax_red":0,"keep_items":512}, {"relax_red":0, "fetch_size":64}]' > gpurun_out/s3d_grid.log 2>&1
ATOS_LIB=$L/libatos_noprobe.so timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{"relax_red":0}, {"relax_red":0,"pipeline":0}]' > gpurun_out/s3d_grid_noprobe.log 2>&1
ATOS_LIB=$L/libatos_keepall.so timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{"relax_red":0,"keep_items":64}, {"relax_red":0,"keep_items":512}, {"relax_red":1,"keep_items":512}]' > gpurun_out/s3d_grid_keepall.log 2>&1
