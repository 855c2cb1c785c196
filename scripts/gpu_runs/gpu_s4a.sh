timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -p no:cacheprovider > gpurun_out/s4a_tests.log 2>&1; echo rc=$? >> gpurun_out/s4a_tests.log
timeout 600 python scripts/exp_pr.py --graph rmat20_pr --configs '[{"relabel":0,"virtual_ranks":8}, {"relabel":0,"virtual_ranks":2}, {"relabel":0,"virtual_ranks":4}]' > gpurun_out/s4a_pr20.log 2>&1
timeout 600 python scripts/exp_bfs.py --graph rmat24 --configs '[{"virtual_ranks":8}, {"virtual_ranks":2}, {"virtual_ranks":4}]' > gpurun_out/s4a_rmat24.log 2>&1
timeout 900 python scripts/exp_pr.py --graph rmat26_pr --reps 1 --configs '[{"relabel":0,"virtual_ranks":8}]' > gpurun_out/s4a_pr26.log 2>&1
