L=$PWD/paper_conf_sc_chenbpbyo22_b200
for rep in 1 2; do
for lib in libatos_head.so libatos.so; do
  echo "== $lib" >> gpurun_out/s3w_ab.log
  ATOS_LIB=$L/$lib timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep cfg >> gpurun_out/s3w_ab.log
  ATOS_LIB=$L/$lib timeout 300 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/s3w_ab.log
  ATOS_LIB=$L/$lib timeout 300 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0}]' 2>&1 | grep cfg >> gpurun_out/s3w_ab.log
done
done
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3w_tests.log 2>&1; echo rc=$? >> gpurun_out/s3w_tests.log
ATOS_SAME_DEVICE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29561 bench.py --gpus 2 --steps 4 --warmup 3 --workload bfs_rmat18 --ctas-per-sm 1 > gpurun_out/s3w_mp_bench.json 2> gpurun_out/s3w_mp_bench.err; echo rc=$? >> gpurun_out/s3w_mp_bench.err
for rep in 1 2; do
  echo "== f4" >> gpurun_out/s3w_ab.log
  ATOS_LIB=$L/libatos_f4.so timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {}]' 2>&1 | grep cfg >> gpurun_out/s3w_ab.log
  ATOS_LIB=$L/libatos_f4.so timeout 300 python scripts/exp_bfs.py --graph rmat26 --configs '[{}]' 2>&1 | grep cfg >> gpurun_out/s3w_ab.log
done
ATOS_LIB=$L/libatos_f4.so timeout 900 python -m pytest tests/test_gpu_bfs.py -m gpu -x -q -p no:cacheprovider -k "filter or rmat or relabel or split" > gpurun_out/s3w_f4_tests.log 2>&1; echo rc=$? >> gpurun_out/s3w_f4_tests.log
ATOS_LOAD_TRACE=1 timeout 300 python scripts/e2e_probe.py > gpurun_out/s3w_e2e.log 2>&1
