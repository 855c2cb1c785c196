timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider -k "not multiprocess" > gpurun_out/gpu_tests23.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests23.log
ATOS_LIB=$PWD/exp_prof.so python scripts/exp_bfs.py --graph rmat24 --configs '[{"pipeline":0}]' 2>&1 | grep -E "PROF cta [01] |cfg" | tail -3 >> gpurun_out/exp23.log
for r in 1 2; do python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"relax_red":0}]' 2>&1 | grep cfg >> gpurun_out/exp23.log; done
python scripts/exp_pr.py >> gpurun_out/exp23.log 2>&1
