# multi-rank instruction fixes (owner_of binary search, destinations present only) A/B vs HEAD;
# pipelined chunk fetch default; stream-ordered load allocations; tests
T=${1:-r2p}
mkdir -p gpurun_out/$T
HL=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_head.so
for lib in new head; do
  L=""; [ $lib = head ] && L=$HL
  ATOS_LIB=$L timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"virtual_ranks":2}, {"virtual_ranks":8}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib /" >> gpurun_out/$T/exp.log
  ATOS_LIB=$L timeout 600 python scripts/exp_pr.py --configs '[{"relabel":0}, {"relabel":0, "virtual_ranks":2}, {"relabel":0, "virtual_ranks":8}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib pr /" >> gpurun_out/$T/exp.log
done
ATOS_LOAD_TRACE=1 timeout 600 python bench.py --steps 2 --warmup 3 --no-pr --north-star 0 --extra-configs 0 --no-cpu-baseline --e2e-steps 10 > gpurun_out/$T/e2e_trace.json 2> gpurun_out/$T/e2e_trace.err
timeout 1800 python -m pytest tests/test_gpu_pq.py tests/test_gpu_bfs.py tests/test_gpu_errors.py tests/test_gpu_multiprocess.py tests/test_gpu_pagerank.py -q -x -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
cut -c1-120 gpurun_out/$T/exp.log; tail -3 gpurun_out/$T/tests.log; grep "chunk" gpurun_out/$T/e2e_trace.err | head -9
python -c "import json; d=json.load(open('gpurun_out/$T/e2e_trace.json')); print(d['e2e'])"
