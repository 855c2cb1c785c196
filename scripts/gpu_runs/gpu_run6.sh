timeout 900 python bench.py > gpurun_out/bench6.json 2> gpurun_out/bench6.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/launches6.csv python bench.py --steps 4 --warmup 3 --no-pr --e2e-steps 0 --no-cpu-baseline --profile-range > gpurun_out/ncu6.log 2>&1
bash scripts/gpu_prof.sh bfs_v3 bfs
