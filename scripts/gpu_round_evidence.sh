# Full evidence pass (one GPU): GPU tests, bench, ncu launch list of the bench's BFS
# step, ncu --set full captures of the BFS (RMAT-24, RMAT-26) and PR workers.
T=${1:-ev}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${T}_smi.txt
timeout 1500 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1; echo rc=$? >> gpurun_out/${T}_tests.log
timeout 900 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/${T}_launches.csv python bench.py --steps 4 --warmup 3 --no-pr --e2e-steps 0 --no-cpu-baseline --north-star 0 --extra-configs 0 --profile-range > gpurun_out/${T}_ncu_launch.log 2>&1
bash scripts/gpu_prof.sh ${T}_bfs bfs
bash scripts/gpu_prof.sh ${T}_bfs26 bfs rmat26
bash scripts/gpu_prof.sh ${T}_pr pr
