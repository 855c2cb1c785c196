# A/B: probe -> next fetch -> finish (working tree) vs HEAD (no pipeline in vis mode ordering), alternating
T=${1:-r2j}
mkdir -p gpurun_out/$T
HL=$PWD/paper_conf_sc_chenbpbyo22_b200/libatos_head.so
for rep in 1 2; do
for gr in rmat24 rmat26; do
  timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{}, {"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/new $gr /" >> gpurun_out/$T/exp.log
  ATOS_LIB=$HL timeout 400 python scripts/exp_bfs.py --graph $gr --configs '[{}, {"pq_delta":1}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/head $gr /" >> gpurun_out/$T/exp.log
done
done
cut -c1-90 gpurun_out/$T/exp.log
