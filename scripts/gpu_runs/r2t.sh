# early next-batch reservation for level buckets (ATOS_NO_PQ_EARLY A/B), tests
T=${1:-r2t}
mkdir -p gpurun_out/$T
for rep in 1 2; do
for v in on off; do
  E=""; [ $v = off ] && E="ATOS_NO_PQ_EARLY=1"
  env $E timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$v rmat24 /" >> gpurun_out/$T/exp.log
  env $E timeout 600 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$v rmat26 /" >> gpurun_out/$T/exp.log
done
done
timeout 1500 python -m pytest tests/test_gpu_pq.py tests/test_gpu_bfs.py tests/test_gpu_queue.py tests/test_gpu_errors.py -q -x -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
cut -c1-120 gpurun_out/$T/exp.log; tail -3 gpurun_out/$T/tests.log
ATOS_LOAD_TRACE=1 timeout 600 python bench.py --steps 2 --warmup 3 --no-pr --north-star 0 --extra-configs 0 --no-cpu-baseline --e2e-steps 10 > gpurun_out/$T/e2e_trace.json 2> gpurun_out/$T/e2e_trace.err
grep "atos load" gpurun_out/$T/e2e_trace.err | grep -v "chunk " | head -40; python -c "import json; d=json.load(open(\"gpurun_out/$T/e2e_trace.json\")); print(d[\"e2e\"])"
