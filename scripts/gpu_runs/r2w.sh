# remote atomics default on virtual ranks, block cache (pool_retain), tests; bench
T=${1:-r2w}
mkdir -p gpurun_out/$T
timeout 2400 python -m pytest tests/test_gpu_pagerank.py tests/test_gpu_errors.py tests/test_gpu_multiprocess.py tests/test_gpu_bfs.py tests/test_gpu_pq.py tests/test_gpu_queue.py tests/test_bench.py -q -x -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
timeout 900 python bench.py > gpurun_out/$T/bench.json 2> gpurun_out/$T/bench.err
tail -3 gpurun_out/$T/tests.log; head -c 300 gpurun_out/$T/bench.json
