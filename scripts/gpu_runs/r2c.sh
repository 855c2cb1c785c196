# staging protocol restored + real agg-off; pq + queue tests; multi-rank A/B
T=${1:-r2c}
mkdir -p gpurun_out/$T
timeout 1500 python -m pytest tests/test_gpu_pq.py tests/test_gpu_queue.py -q -x > gpurun_out/$T/new_tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/new_tests.log
timeout 1500 python -m pytest tests/test_gpu_bfs.py tests/test_gpu_pagerank.py tests/test_gpu_errors.py tests/test_gpu_multiprocess.py -q -x -k "virtual or multi or combining or processes or config4 or injected or tiny" > gpurun_out/$T/multi_tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/multi_tests.log
for lib in libatos_bf97c53.so libatos.so; do
  for vr in 2 8; do
    echo "== $lib bfs vr$vr" >> gpurun_out/$T/ab.log
    ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/$lib timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs "[{\"virtual_ranks\":$vr}, {\"virtual_ranks\":$vr, \"agg_enabled\":0}]" 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/ab.log
    echo "== $lib pr vr$vr" >> gpurun_out/$T/ab.log
    ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/$lib timeout 300 python scripts/exp_pr.py --graph rmat20_pr --configs "[{\"virtual_ranks\":$vr}, {\"virtual_ranks\":$vr, \"agg_enabled\":0}]" 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/ab.log
  done
done
tail -5 gpurun_out/$T/new_tests.log gpurun_out/$T/multi_tests.log
