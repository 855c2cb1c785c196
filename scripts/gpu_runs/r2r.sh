# multi-rank: inbound rings per rank x channel packets x packet size (virtual ranks), incremental channel walk
T=${1:-r2r}
mkdir -p gpurun_out/$T
for R in 8 32; do
ATOS_INBOUND_RINGS=$R timeout 900 python scripts/exp_pr.py --reps 2 --configs '[{"relabel":0, "virtual_ranks":2, "channel_packets":4096}, {"relabel":0, "virtual_ranks":2, "channel_packets":4096, "agg_batch_msgs":1024}, {"relabel":0, "virtual_ranks":8, "channel_packets":4096}, {"relabel":0, "virtual_ranks":8, "channel_packets":4096, "agg_batch_msgs":1024}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/R$R pr /" >> gpurun_out/$T/exp.log
ATOS_INBOUND_RINGS=$R timeout 900 python scripts/exp_bfs.py --graph rmat24 --configs '[{"virtual_ranks":2, "channel_packets":4096}, {"virtual_ranks":2, "channel_packets":4096, "agg_batch_msgs":1024}, {"virtual_ranks":8, "channel_packets":4096}, {"virtual_ranks":8, "channel_packets":4096, "agg_batch_msgs":1024}]' 2>&1 | grep -E "cfg|Error" | sed "s/^/R$R bfs /" >> gpurun_out/$T/exp.log
done
cut -c1-150 gpurun_out/$T/exp.log
