timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s3g_tests.log 2>&1; echo rc=$? >> gpurun_out/s3g_tests.log
bash scripts/gpu_prof.sh s3g_pr_vr8 pr rmat20_pr '{"relabel":0,"virtual_ranks":8}'
