timeout 300 python scripts/discrete_probe.py > gpurun_out/s3i_discrete.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3i_tests.log 2>&1; echo rc=$? >> gpurun_out/s3i_tests.log
timeout 400 ./scripts/queue_micro 20 > gpurun_out/s3i_queue_micro.jsonl 2> gpurun_out/s3i_queue_micro.err
