python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_bfs.py tests/test_gpu_pagerank.py tests/test_gpu_multiprocess.py -q -x -k "virtual or multi or combining or relabel or processes or row_splitting or config4" 2>&1 | tail -3
for vr in 1 2 4 8; do timeout 300 python scripts/exp_bfs.py --graph rmat24 --configs "[{\"virtual_ranks\":$vr}, {\"virtual_ranks\":$vr, \"agg_enabled\":0}]" 2>&1 | grep cfg; done
for vr in 1 2 8; do timeout 300 python scripts/exp_pr.py --graph rmat20_pr --configs "[{\"relabel\":0, \"virtual_ranks\":$vr}, {\"relabel\":0, \"virtual_ranks\":$vr, \"agg_enabled\":0}]" 2>&1 | grep cfg; done
