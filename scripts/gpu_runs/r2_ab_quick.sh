# quick A/B of BFS configs on rmat24 / rmat26 (+ optional env variants): bash r2_ab_quick.sh <tag> '<configs json>' [graphs]
T=$1; CF=$2; GRS=${3:-"rmat24 rmat26"}
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/$T/build.log 2>&1
for gr in $GRS; do
  timeout 600 python scripts/exp_bfs.py --graph $gr --configs "$CF" >> gpurun_out/$T/ab.log 2>&1
done
grep -E "cfg|graph|Error" gpurun_out/$T/ab.log
