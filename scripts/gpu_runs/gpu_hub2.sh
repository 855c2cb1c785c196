timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/hub2_tests.log 2>&1; echo rc=$? >> gpurun_out/hub2_tests.log
bash scripts/gpu_prof.sh hubon bfs rmat24 '{}'
bash scripts/gpu_prof.sh huboff bfs rmat24 '{"relabel":1,"hub_cache":0}'
