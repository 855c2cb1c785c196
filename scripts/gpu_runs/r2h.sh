# relax_vis with batched atomics + warp cursor for long-chunk rows + auto level buckets: tests + timing
T=${1:-r2h}
mkdir -p gpurun_out/$T
for gr in rmat24 rmat26; do
  timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{}, {"pq_delta":0}, {"pq_delta":1}, {}, {"pq_delta":0}, {"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$gr /" >> gpurun_out/$T/exp.log
done
timeout 1500 python -m pytest tests/test_gpu_pq.py tests/test_gpu_bfs.py tests/test_gpu_queue.py -q -x -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
bash scripts/gpu_prof.sh ${T}_bfs26 bfs rmat26
cat gpurun_out/$T/exp.log; tail -3 gpurun_out/$T/tests.log
