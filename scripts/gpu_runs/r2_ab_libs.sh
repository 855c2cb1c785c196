# A/B of variant libraries: bash r2_ab_libs.sh <tag> '<configs json>' '<graphs>' lib1 lib2 ...
T=$1; CF=$2; GRS=$3; shift 3
mkdir -p gpurun_out/$T
for rep in 1 2; do
for lib in "$@"; do
  for gr in $GRS; do
    echo "== $lib $gr" >> gpurun_out/$T/ab.log
    ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/$lib timeout 600 python scripts/exp_bfs.py --graph $gr --configs "$CF" 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/ab.log
  done
done
done
cat gpurun_out/$T/ab.log
