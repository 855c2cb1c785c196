# A/B: claim at pop (ATOS_VIS_CLAIM) vs discoverer atomicOr, RMAT-24/26 level buckets; parity with the switch
T=${1:-r2k}
mkdir -p gpurun_out/$T
for rep in 1 2; do
for gr in rmat26 rmat24; do
  timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/base $gr /" >> gpurun_out/$T/exp.log
  ATOS_VIS_CLAIM=1 timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/claim $gr /" >> gpurun_out/$T/exp.log
done
done
ATOS_VIS_CLAIM=1 timeout 900 python -m pytest tests/test_gpu_pq.py -q -x -p no:cacheprovider -k "not virtual" > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
ATOS_VIS_CLAIM=1 timeout 900 python -m pytest tests/test_gpu_bfs.py -q -x -p no:cacheprovider -k "rmat26 or rmat24_config2_full_size" >> gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
cut -c1-120 gpurun_out/$T/exp.log; tail -5 gpurun_out/$T/tests.log
