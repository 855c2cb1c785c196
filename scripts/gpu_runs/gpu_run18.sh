E='python scripts/exp_bfs.py --graph rmat24 --configs [{}]'
for lib in exp_prof.so exp_profA.so; do echo "== $lib" >> gpurun_out/exp18.log; ATOS_LIB=$PWD/$lib $E 2>&1 | grep -E "PROF cta 0|cfg" | tail -3 >> gpurun_out/exp18.log; done
for r in 1 2; do for lib in paper_conf_sc_chenbpbyo22_b200/libatos.so exp_A.so; do echo "== $lib" >> gpurun_out/exp18.log; ATOS_LIB=$PWD/$lib python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"relax_red":1}]' 2>&1 | grep cfg >> gpurun_out/exp18.log; done; done
