python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"fetch_size":128}, {"fetch_size":64}, {"ctas_per_sm":1}]' > gpurun_out/exp2.log 2>&1
python scripts/exp_bfs.py --graph path1000000 --configs '[{}]' >> gpurun_out/exp2.log 2>&1
python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' >> gpurun_out/exp2.log 2>&1
timeout 900 ncu --set full --replay-mode application --profile-from-start off --clock-control none --import-source on -k regex:worker_kernel -c 1 -o gpurun_out/prof_bfs python scripts/prof_worker.py --app bfs > gpurun_out/ncu_bfs.log 2>&1
