# multi-rank BFS: remote atomicMin + activations (ATOS_BFS_RATOM) vs messages; parity with the switch
T=${1:-r2x}
mkdir -p gpurun_out/$T
for rep in 1 2; do
for v in msg ratom; do
  E=""; [ $v = ratom ] && E="ATOS_BFS_RATOM=1"
  env $E timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"virtual_ranks":2}, {"virtual_ranks":4}, {"virtual_ranks":8}, {"virtual_ranks":8, "pq_delta":1}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$v /" >> gpurun_out/$T/exp.log
  env $E timeout 600 python scripts/exp_bfs.py --graph grid4900 --configs '[{"virtual_ranks":4}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$v grid /" >> gpurun_out/$T/exp.log
done
done
ATOS_BFS_RATOM=1 timeout 1500 python -m pytest tests/test_gpu_bfs.py tests/test_gpu_pq.py -q -x -p no:cacheprovider -k "virtual or ranks or vr" > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
cut -c1-160 gpurun_out/$T/exp.log; tail -3 gpurun_out/$T/tests.log
