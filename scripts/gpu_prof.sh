# usage: bash scripts/gpu_prof.sh <tag> <app> [graph] [cfg-json]
TAG=$1; APP=$2; GRAPH=${3:-}; CFG=${4:-"{}"}
ARGS="--app $APP"; [ -n "$GRAPH" ] && ARGS="$ARGS --graph $GRAPH"
timeout 1200 ncu --set full --replay-mode application --profile-from-start off --clock-control none --import-source on -k regex:worker_kernel -c 1 -o gpurun_out/prof_$TAG python scripts/prof_worker.py $ARGS --cfg "$CFG" > gpurun_out/ncu_$TAG.log 2>&1
tail -3 gpurun_out/ncu_$TAG.log
