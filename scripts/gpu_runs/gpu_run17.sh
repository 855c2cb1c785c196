timeout 600 python -m torch.distributed.run --standalone --nproc-per-node 2 scripts/mp_same_gpu.py > gpurun_out/mp1.log 2>&1; echo rc=$? >> gpurun_out/mp1.log
for r in 1 2; do
python scripts/exp_bfs.py --graph rmat24 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/exp17.log
ATOS_LIB=$PWD/exp_l1.so python scripts/exp_bfs.py --graph rmat24 --configs '[{"fetch_size":512}]' 2>&1 | grep cfg >> gpurun_out/exp17.log
done
