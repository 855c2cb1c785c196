# confirmation at the round's last commit: GPU tests, smoke, bench
T=${1:-r2final}
mkdir -p gpurun_out/$T
timeout 2700 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/$T/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/$T/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/$T/smoke.log
timeout 900 python bench.py > gpurun_out/$T/bench.json 2> gpurun_out/$T/bench.err
tail -3 gpurun_out/$T/pytest.log gpurun_out/$T/smoke.log; head -c 300 gpurun_out/$T/bench.json
