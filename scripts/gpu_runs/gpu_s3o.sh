ATOS_LOAD_TRACE=1 timeout 600 python scripts/load_timing.py rmat24 > gpurun_out/s3o_load.log 2>&1
bash scripts/gpu_prof.sh s3o_pr_vr8 pr rmat20_pr '{"relabel":0,"virtual_ranks":8}'
