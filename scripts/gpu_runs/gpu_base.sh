# Re-establish the current numbers on a fresh box: GPU tests + bench.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > gpurun_out/base_smi.txt 2>&1
nproc >> gpurun_out/base_smi.txt
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/base_tests.log 2>&1; echo rc=$? >> gpurun_out/base_tests.log
timeout 900 python bench.py > gpurun_out/base_bench.json 2> gpurun_out/base_bench.err
