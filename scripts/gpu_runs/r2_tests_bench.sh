# round-2 evidence pass: GPU tests, smoke, bench (N=1), reference arm
T=${1:-r2a}
mkdir -p gpurun_out/$T
nproc > gpurun_out/$T/host.txt; lscpu | grep -E "Model name|^CPU\(s\)|Thread|Socket" >> gpurun_out/$T/host.txt
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv >> gpurun_out/$T/host.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/$T/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x --durations=25 > gpurun_out/$T/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/$T/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/$T/bench.json 2> gpurun_out/$T/bench.err
tail -3 gpurun_out/$T/pytest.log
