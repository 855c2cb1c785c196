# usage: bash scripts/gpu_exp.sh <tag> <run-tests 0/1> <graph> '<configs json>' [<graph> '<configs>' ...]
TAG=$1; T=$2; shift 2
if [ "$T" = "1" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/${TAG}_tests.log 2>&1; echo rc=$? >> gpurun_out/${TAG}_tests.log
fi
while [ $# -ge 2 ]; do
  timeout 900 python scripts/exp_bfs.py --graph $1 --configs "$2" >> gpurun_out/${TAG}_exp.log 2>&1
  shift 2
done
