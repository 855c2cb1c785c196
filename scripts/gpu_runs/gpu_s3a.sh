# Session-3 baseline on HEAD: gpu tests, bench, launch list.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/s3a_smi.txt
timeout 1500 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider --durations=15 > gpurun_out/s3a_tests.log 2>&1; echo rc=$? >> gpurun_out/s3a_tests.log
timeout 900 python bench.py > gpurun_out/s3a_bench.json 2> gpurun_out/s3a_bench.err
