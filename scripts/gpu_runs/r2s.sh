# wide inbound poll vs one-by-one (variant), new channel defaults; multi-rank tests
T=${1:-r2s}
mkdir -p gpurun_out/$T
NL=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_narrow.so
for rep in 1 2; do
for lib in wide narrow; do
  L=""; [ $lib = narrow ] && L=$NL
  ATOS_LIB=$L timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"virtual_ranks":2}, {"virtual_ranks":8}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib /" >> gpurun_out/$T/exp.log
  ATOS_LIB=$L timeout 600 python scripts/exp_pr.py --reps 2 --configs '[{"relabel":0, "virtual_ranks":2}, {"relabel":0, "virtual_ranks":4}, {"relabel":0, "virtual_ranks":8}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib pr /" >> gpurun_out/$T/exp.log
done
done
timeout 1800 python -m pytest tests/test_gpu_bfs.py tests/test_gpu_pagerank.py tests/test_gpu_multiprocess.py tests/test_gpu_errors.py tests/test_gpu_pq.py tests/test_bench.py -q -x -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
cut -c1-130 gpurun_out/$T/exp.log; tail -3 gpurun_out/$T/tests.log
