# ncu --set full of one worker launch per variant: bash r2_prof.sh <tag> <graph> <cfgjson> [<cfgjson> ...]
T=$1; GR=$2; shift 2
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/$T/build.log 2>&1
i=0
for CFG in "$@"; do
  timeout 1500 ncu --set full --replay-mode application --profile-from-start off --clock-control none --import-source on \
    -k regex:worker_kernel -c 1 -o gpurun_out/$T/prof_$i python scripts/prof_worker.py --app bfs --graph $GR --cfg "$CFG" > gpurun_out/$T/ncu_$i.log 2>&1
  echo "$i $CFG" >> gpurun_out/$T/variants.txt
  i=$((i+1))
done
ls -la gpurun_out/$T
