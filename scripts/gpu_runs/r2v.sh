# multi-rank PR: remote atomics + activation messages (ATOS_PR_RATOM) vs delta messages; parity
T=${1:-r2v}
mkdir -p gpurun_out/$T
for rep in 1 2; do
for v in msg ratom; do
  E=""; [ $v = ratom ] && E="ATOS_PR_RATOM=1"
  env $E timeout 600 python scripts/exp_pr.py --reps 2 --configs '[{"relabel":0, "virtual_ranks":2}, {"relabel":0, "virtual_ranks":4}, {"relabel":0, "virtual_ranks":8}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$v pr /" >> gpurun_out/$T/exp.log
done
done
ATOS_PR_RATOM=1 timeout 1500 python -m pytest tests/test_gpu_pagerank.py -q -x -p no:cacheprovider > gpurun_out/$T/tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/tests.log
cut -c1-200 gpurun_out/$T/exp.log; tail -3 gpurun_out/$T/tests.log
