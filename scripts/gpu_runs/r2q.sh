# multi-rank channel capacity / packet size sweep (virtual ranks): PR RMAT-20 and BFS RMAT-24
T=${1:-r2q}
mkdir -p gpurun_out/$T
timeout 900 python scripts/exp_pr.py --reps 2 --configs '[{"relabel":0, "virtual_ranks":2}, {"relabel":0, "virtual_ranks":2, "channel_packets":4096}, {"relabel":0, "virtual_ranks":2, "channel_packets":16384}, {"relabel":0, "virtual_ranks":2, "channel_packets":4096, "agg_batch_msgs":1024}, {"relabel":0, "virtual_ranks":8}, {"relabel":0, "virtual_ranks":8, "channel_packets":4096}, {"relabel":0, "virtual_ranks":8, "channel_packets":16384}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/pr /" >> gpurun_out/$T/exp.log
timeout 900 python scripts/exp_bfs.py --graph rmat24 --configs '[{"virtual_ranks":2}, {"virtual_ranks":2, "channel_packets":4096}, {"virtual_ranks":2, "channel_packets":16384}, {"virtual_ranks":8}, {"virtual_ranks":8, "channel_packets":4096}, {"virtual_ranks":8, "channel_packets":16384}, {"virtual_ranks":8, "agg_batch_msgs":64}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/bfs /" >> gpurun_out/$T/exp.log
cut -c1-150 gpurun_out/$T/exp.log
