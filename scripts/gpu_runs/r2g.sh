# FIFO vs visited-bitmap level buckets (pq_delta=1) on RMAT-24/26; ncu of the RMAT-26 vis worker
T=${1:-r2g}
mkdir -p gpurun_out/$T
for gr in rmat24 rmat26; do
  timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{}, {"pq_delta":1}, {}, {"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/exp.log
done
bash scripts/gpu_prof.sh ${T}_bfs26vis bfs rmat26 '{"pq_delta":1}'
bash scripts/gpu_prof.sh ${T}_bfs24vis bfs rmat24 '{"pq_delta":1}'
cat gpurun_out/$T/exp.log
