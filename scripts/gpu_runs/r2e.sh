# visited-bitmap level-synchronous mode: tests + timing
T=${1:-r2e}
mkdir -p gpurun_out/$T
timeout 1500 python -m pytest tests/test_gpu_pq.py tests/test_gpu_queue.py -q > gpurun_out/$T/new_tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/new_tests.log
for gr in rmat24 rmat26; do
  timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{}, {"pq_delta":1}, {"pq_delta":2}]' 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/exp.log
  ATOS_NO_VIS=1 timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" | sed 's/^/NO_VIS /' >> gpurun_out/$T/exp.log
done
timeout 300 python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"pq_delta":1}, {"pq_delta":64}]' 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/exp.log
timeout 1500 python -m pytest tests/test_gpu_bfs.py -q -x > gpurun_out/$T/bfs_tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/bfs_tests.log
tail -3 gpurun_out/$T/new_tests.log gpurun_out/$T/bfs_tests.log
