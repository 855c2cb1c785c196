# N4 queue sweep on libatos's ring code + compute-sanitizer (racecheck, synccheck, memcheck) on tiny solves
T=${1:-r2n}
mkdir -p gpurun_out/$T
timeout 900 python scripts/qbench_sweep.py > gpurun_out/$T/qbench_sweep.jsonl 2> gpurun_out/$T/qbench_sweep.err
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 30 --error-exitcode 9 python scripts/sanitize_tiny.py > gpurun_out/$T/san_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/$T/san_$tool.log
done
wc -l gpurun_out/$T/qbench_sweep.jsonl; tail -4 gpurun_out/$T/san_*.log
bash scripts/gpu_prof.sh ${T}_bfs24vr8 bfs rmat24 '{"virtual_ranks":8}'
bash scripts/gpu_prof.sh ${T}_pr20vr2 pr rmat20_pr '{"virtual_ranks":2, "relabel":0}'
