# Full evidence pass: GPU tests, bench, launch list, ncu full capture of the BFS and PR workers.
set -x
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/ev_tests.log 2>&1; echo rc=$? >> gpurun_out/ev_tests.log
timeout 900 python bench.py > gpurun_out/ev_bench.json 2> gpurun_out/ev_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/ev_launches.csv python bench.py --steps 4 --warmup 3 --no-pr --e2e-steps 0 --no-cpu-baseline --profile-range > gpurun_out/ev_ncu_launch.log 2>&1
bash scripts/gpu_prof.sh ev_bfs bfs
bash scripts/gpu_prof.sh ev_pr pr
