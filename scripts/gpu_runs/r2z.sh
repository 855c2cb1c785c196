# final round-2 evidence pass: GPU tests, smoke, bench (N=1), reference arm, launch list, ncu of the
# BFS + PR workers (summaries made on the box; only the RMAT-24 BFS report is brought back: <= 64 MiB)
T=${1:-r2z2}
mkdir -p gpurun_out/$T
nproc > gpurun_out/$T/host.txt; lscpu | grep -E "Model name|^CPU\(s\)|Thread|Socket" >> gpurun_out/$T/host.txt
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv >> gpurun_out/$T/host.txt
timeout 2700 python -m pytest tests -m gpu -q -x --durations=30 -p no:cacheprovider > gpurun_out/$T/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/$T/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/$T/smoke.log
timeout 900 python bench.py > gpurun_out/$T/bench.json 2> gpurun_out/$T/bench.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/$T/bench_reference.json 2> gpurun_out/$T/bench_reference.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/$T/launches.csv python bench.py --steps 4 --warmup 3 --no-pr --e2e-steps 0 --no-cpu-baseline --north-star 0 --extra-configs 0 --profile-range > gpurun_out/$T/ncu_launch.log 2>&1
prof() {   # tag app graph cfg
  bash scripts/gpu_prof.sh ${T}_$1 $2 $3 "$4"
  python scripts/ncu_summary.py gpurun_out/prof_${T}_$1.ncu-rep 25 > gpurun_out/$T/ncu_$1_summary.txt 2>&1
  python scripts/ncu_sectors.py gpurun_out/prof_${T}_$1.ncu-rep 30 stall > gpurun_out/$T/ncu_$1_lines.txt 2>&1
  python scripts/ncu_sectors.py gpurun_out/prof_${T}_$1.ncu-rep 30 inst > gpurun_out/$T/ncu_$1_inst.txt 2>&1
}
prof bfs24 bfs rmat24 '{}'
prof bfs26 bfs rmat26 '{}'; rm -f gpurun_out/prof_${T}_bfs26.ncu-rep
prof pr20 pr rmat20_pr '{}'; rm -f gpurun_out/prof_${T}_pr20.ncu-rep
prof pr20vr8 pr rmat20_pr '{"virtual_ranks":8, "relabel":0}'; rm -f gpurun_out/prof_${T}_pr20vr8.ncu-rep
prof bfs24vr8 bfs rmat24 '{"virtual_ranks":8}'; rm -f gpurun_out/prof_${T}_bfs24vr8.ncu-rep
du -sh gpurun_out
tail -3 gpurun_out/$T/pytest.log gpurun_out/$T/smoke.log; head -c 400 gpurun_out/$T/bench.json
