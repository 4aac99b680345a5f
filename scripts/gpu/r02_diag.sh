timeout 600 python scripts/walker_diag.py 6 > gpurun_out/walker_diag.log 2>&1; echo rc=$?
cat gpurun_out/walker_diag.log | tail -60
