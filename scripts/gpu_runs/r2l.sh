# FIFO vs level buckets (claim at pop) across RMAT scales: the auto threshold; pq tests
T=${1:-r2l}
mkdir -p gpurun_out/$T
for gr in kron12 rmat16 rmat18 rmat20 rmat22 rmat23 rmat24 rmat25; do
  timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{"pq_delta":0}, {"pq_delta":1}, {"pq_delta":0}, {"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$gr /" >> gpurun_out/$T/exp.log
done
timeout 900 python -m pytest tests/test_gpu_pq.py -q -x -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
cut -c1-110 gpurun_out/$T/exp.log; tail -3 gpurun_out/$T/tests.log
