ATOS_LOAD_TRACE=1 timeout 300 python scripts/e2e_probe.py > gpurun_out/s3x_e2e.log 2>&1
ATOS_LOAD_STREAMED=0 ATOS_LOAD_TRACE=1 timeout 300 python scripts/e2e_probe.py > gpurun_out/s3x_e2e_nostream.log 2>&1
