# BFS remote atomics vs depth messages at 2 / 3 / 4 virtual ranks, alternating, same box
T=${1:-r2y}
mkdir -p gpurun_out/$T
for rep in 1 2 3; do
for v in msg ratom; do
  E="ATOS_BFS_NORATOM=1"; [ $v = ratom ] && E="ATOS_UNUSED=1"
  env $E timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"virtual_ranks":2}, {"virtual_ranks":3}, {"virtual_ranks":4}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$v /" >> gpurun_out/$T/exp.log
done
done
cut -c1-100 gpurun_out/$T/exp.log
