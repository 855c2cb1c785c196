# N1 priority-queue tests + multi-rank A/B of variant libraries (virtual ranks)
T=${1:-r2b}
mkdir -p gpurun_out/$T
timeout 900 python -m pytest tests/test_gpu_pq.py -q -x > gpurun_out/$T/pq_tests.log 2>&1; echo "rc=$?" >> gpurun_out/$T/pq_tests.log
for lib in libatos_bf97c53.so libatos_de6adde.so libatos.so; do
  for vr in 2 8; do
    echo "== $lib bfs vr$vr" >> gpurun_out/$T/ab.log
    ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/$lib timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs "[{\"virtual_ranks\":$vr}]" 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/ab.log
    echo "== $lib pr vr$vr" >> gpurun_out/$T/ab.log
    ATOS_LIB=$PWD/paper_conf_sc_chenbpbyo22_b200/$lib timeout 300 python scripts/exp_pr.py --graph rmat20_pr --configs "[{\"virtual_ranks\":$vr}]" 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/ab.log
  done
done
for d in 1 2 4; do
  for vr in 1 2 8; do
    timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs "[{\"virtual_ranks\":$vr, \"pq_delta\":$d}]" 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/pq_exp.log
  done
done
timeout 300 python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"pq_delta":1}, {"pq_delta":16}, {"pq_delta":256}, {"pq_delta":4096}]' 2>&1 | grep -E "cfg|Error" >> gpurun_out/$T/pq_exp.log
cat gpurun_out/$T/pq_tests.log | tail -15
