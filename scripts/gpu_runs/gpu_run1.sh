set -x
timeout 600 python -m pytest tests -m gpu -x -q -k slow --timeout 500 -p no:cacheprovider > gpurun_out/gpu_slow.log 2>&1; echo rc=$? >> gpurun_out/gpu_slow.log
timeout 600 python bench.py > gpurun_out/bench1.json 2> gpurun_out/bench1.err; echo rc=$? >> gpurun_out/bench1.err
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches1.csv python bench.py --steps 2 --warmup 3 --no-pr --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu1.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:worker_kernel -s 6 -c 1 -o gpurun_out/prof_bfs python bench.py --steps 2 --warmup 3 --no-pr --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu2.log 2>&1
