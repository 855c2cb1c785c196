# load-phase timing + fresh launch list + ncu full captures of the current workers
ATOS_LOAD_TRACE=1 timeout 600 python scripts/load_timing.py rmat24 > gpurun_out/s3b_load.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/s3b_launches.csv python bench.py --steps 4 --warmup 3 --no-pr --e2e-steps 0 --no-cpu-baseline --north-star 0 --profile-range > gpurun_out/s3b_ncu_launch.log 2>&1
bash scripts/gpu_prof.sh s3b_bfs bfs
bash scripts/gpu_prof.sh s3b_pr pr
