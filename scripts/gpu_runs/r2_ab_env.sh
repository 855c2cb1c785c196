# A/B over an environment variable: bash r2_ab_env.sh <tag> VAR '<values>' '<configs json>' '<graphs>'
T=$1; VAR=$2; VALS=$3; CF=$4; GRS=$5
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/$T/build.log 2>&1
for rep in 1 2; do
for v in $VALS; do
  for gr in $GRS; do
    echo "== $VAR=$v $gr" >> gpurun_out/$T/ab.log
    env $VAR=$v timeout 600 python scripts/exp_bfs.py --graph $gr --configs "$CF" 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/ab.log
  done
done
done
cat gpurun_out/$T/ab.log
