timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3y_tests.log 2>&1; echo rc=$? >> gpurun_out/s3y_tests.log
ATOS_LOAD_TRACE=1 timeout 300 python scripts/e2e_probe.py > gpurun_out/s3y_e2e.log 2>&1
timeout 900 python bench.py --north-star 0 --extra-configs 0 > gpurun_out/s3y_bench.json 2> gpurun_out/s3y_bench.err
