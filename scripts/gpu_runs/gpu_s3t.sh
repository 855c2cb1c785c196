timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider -k "full_size" --durations=10 > gpurun_out/s3t_tests.log 2>&1; echo rc=$? >> gpurun_out/s3t_tests.log
free -g > gpurun_out/s3t_free.txt; nproc >> gpurun_out/s3t_free.txt
