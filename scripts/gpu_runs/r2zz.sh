# A/B: long-row threshold kLong 32 / 64 (default) / 128, single-rank BFS RMAT-24 / RMAT-26
T=${1:-r2zz2}
mkdir -p gpurun_out/$T
P=$PWD/paper_conf_sc_chenbpbyo22_b200
for rep in 1 2; do
for lib in libatos libatos_kl128 libatos_kl192 libatos_kl256; do
  ATOS_LIB=$P/$lib.so timeout 400 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib rmat24 /" >> gpurun_out/$T/exp.log
  ATOS_LIB=$P/$lib.so timeout 400 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/$lib rmat26 /" >> gpurun_out/$T/exp.log
done
done
