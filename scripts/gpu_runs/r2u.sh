# A/B: ballot-per-slot append + row_ptr reuse at load (working tree) vs HEAD; BFS 1 rank + PR; e2e
T=${1:-r2u}
mkdir -p gpurun_out/$T
HL=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_head.so
for rep in 1 2; do
for lib in new head; do
  L=""; [ $lib = head ] && L=$HL
  ATOS_LIB=$L timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"pq_delta":0}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib rmat24 /" >> gpurun_out/$T/exp.log
  ATOS_LIB=$L timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib rmat26 /" >> gpurun_out/$T/exp.log
  ATOS_LIB=$L timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib grid /" >> gpurun_out/$T/exp.log
  ATOS_LIB=$L timeout 600 python scripts/exp_pr.py --reps 2 --configs '[{"relabel":0}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib pr /" >> gpurun_out/$T/exp.log
done
done
ATOS_LOAD_TRACE=1 timeout 600 python bench.py --steps 2 --warmup 3 --no-pr --north-star 0 --extra-configs 0 --no-cpu-baseline --e2e-steps 10 > gpurun_out/$T/e2e_trace.json 2> gpurun_out/$T/e2e_trace.err
timeout 1500 python -m pytest tests/test_gpu_pq.py tests/test_gpu_bfs.py -q -x -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
cut -c1-110 gpurun_out/$T/exp.log; tail -3 gpurun_out/$T/tests.log
python -c "import json; d=json.load(open('gpurun_out/$T/e2e_trace.json')); print(d['e2e'])"
