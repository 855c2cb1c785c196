# A/B: chunk pipeline off / fetch-first / probe-first (variant libraries), RMAT-24/26 (level buckets) and FIFO RMAT-24
T=${1:-r2o}
mkdir -p gpurun_out/$T
P=$PWD/paper_conf_sc_chenbpbyo22_b200
for rep in 1 2; do
for lib in libatos libatos_pipe1 libatos_pipe2; do
  for gr in rmat24 rmat26; do
    ATOS_LIB=$P/$lib.so timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{}, {"pq_delta":0}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib $gr /" >> gpurun_out/$T/exp.log
  done
done
done
cut -c1-110 gpurun_out/$T/exp.log
for gr in rmat24 rmat26; do
  ATOS_HUB_DBG=7 timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{}, {}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/nohub $gr /" >> gpurun_out/$T/exp.log
done
cut -c1-110 gpurun_out/$T/exp.log | grep nohub
# e2e load outliers: phase trace of 10 load/solve/free steps
ATOS_LOAD_TRACE=1 timeout 600 python bench.py --steps 2 --warmup 3 --no-pr --north-star 0 --extra-configs 0 --no-cpu-baseline --e2e-steps 10 > gpurun_out/$T/e2e_trace.json 2> gpurun_out/$T/e2e_trace.err
grep "atos load" gpurun_out/$T/e2e_trace.err | sort | awk '{print $3}' | uniq -c | head; python -c "import json; d=json.load(open('gpurun_out/$T/e2e_trace.json')); print(d['e2e'])"
