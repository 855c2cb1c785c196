# pipelined chunk fetch: timing + tests
T=${1:-r2i}
mkdir -p gpurun_out/$T
for gr in rmat24 rmat26 grid4900; do
  timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{}, {}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$gr /" >> gpurun_out/$T/exp.log
done
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/rmat24 /" >> gpurun_out/$T/exp.log
timeout 1500 python -m pytest tests/test_gpu_pq.py tests/test_gpu_bfs.py -q -x -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
cat gpurun_out/$T/exp.log; tail -3 gpurun_out/$T/tests.log
