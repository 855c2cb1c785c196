for a in "1 0" "0 1024" "1 -1"; do timeout 120 python scripts/dbg_hub.py $a >> gpurun_out/dbg1.log 2>&1; done
timeout 600 compute-sanitizer --tool memcheck --print-limit 5 python scripts/dbg_hub.py 1 -1 >> gpurun_out/dbg1.log 2>&1
