# A/B: lean single-rank BFS expansion (atos_bfs1.cuh) vs the generic one (ATOS_BFS_V1)
T=${1:-r2b}
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/$T/build.log 2>&1
for gr in rmat24 rmat26 grid4900; do
  timeout 600 python scripts/exp_bfs.py --graph $gr --configs '[{}, {"hub_cache":0}, {"hub_cache":4194304}, {}]' >> gpurun_out/$T/ab.log 2>&1
  ATOS_BFS_V1=1 timeout 600 python scripts/exp_bfs.py --graph $gr --configs '[{}, {}]' 2>&1 | sed 's/"cfg": {/"cfg": {"V1":1, /' >> gpurun_out/$T/ab.log
done
timeout 1200 python -m pytest tests/test_gpu_bfs.py -q -x -k "bfs1 or hub_cache or relabel or runtime or rmat24_config2_full_size or rmat26" > gpurun_out/$T/pytest.log 2>&1
echo "rc=$?" >> gpurun_out/$T/pytest.log
cat gpurun_out/$T/ab.log | grep -E "cfg|graph"
tail -3 gpurun_out/$T/pytest.log
timeout 900 python -m pytest tests/test_bench.py tests/test_gpu_errors.py -q -x > gpurun_out/$T/pytest2.log 2>&1
tail -3 gpurun_out/$T/pytest2.log
timeout 1200 python bench.py > gpurun_out/$T/bench.json 2> gpurun_out/$T/bench.err
tail -2 gpurun_out/$T/bench.err
