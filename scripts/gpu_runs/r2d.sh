# pq (CAS reservation near empty) tests + redundancy table + ncu of the BFS worker
T=${1:-r2d}
mkdir -p gpurun_out/$T
timeout 1500 python -m pytest tests/test_gpu_pq.py tests/test_gpu_queue.py -q > gpurun_out/$T/new_tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/new_tests.log
for vr in 1 2 4 8; do
  timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs "[{\"virtual_ranks\":$vr}, {\"virtual_ranks\":$vr, \"pq_delta\":1}, {\"virtual_ranks\":$vr, \"pq_delta\":2}]" 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/pq_exp.log
done
timeout 300 python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"keep_items":0}, {"pq_delta":1}, {"pq_delta":64}, {"pq_delta":1024}]' 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/pq_exp.log
timeout 300 python scripts/exp_bfs.py --graph rmat26 --configs '[{}, {"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/pq_exp.log
bash scripts/gpu_prof.sh ${T}_bfs24 bfs rmat24
bash scripts/gpu_prof.sh ${T}_bfs26 bfs rmat26
tail -3 gpurun_out/$T/new_tests.log
