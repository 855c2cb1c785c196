python -c "import torch;p=torch.cuda.get_device_properties(0);print('persist', getattr(p,'persisting_l2_cache_max_size',None))" > gpurun_out/exp4.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests4.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests4.log
python scripts/exp_bfs.py --graph rmat24 --configs '[{}, {"keep_items":0}, {"l2_persist":0}, {"keep_items":0, "l2_persist":0}]' >> gpurun_out/exp4.log 2>&1
python scripts/exp_bfs.py --graph grid4900 --configs '[{}, {"keep_items":0}]' >> gpurun_out/exp4.log 2>&1
