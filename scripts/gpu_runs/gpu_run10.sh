for v in 4 12 16; do echo "== kU=$v" >> gpurun_out/exp10.log; ATOS_LIB=$PWD/exp_ku$v.so python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' >> gpurun_out/exp10.log 2>&1; done
echo "== kU=8" >> gpurun_out/exp10.log; python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' >> gpurun_out/exp10.log 2>&1
