cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 1 -c 1 -o gpurun_out/prof_det python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --variants det32 > gpurun_out/ncu_det.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 1 -c 1 -o gpurun_out/prof_par python scripts/diag.py --graph road:4900 --roots 1 --reps 1 --variants h2c2pb1 > gpurun_out/ncu_par.log 2>&1
tail -2 gpurun_out/ncu_det.log gpurun_out/ncu_par.log
