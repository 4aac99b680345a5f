cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r01
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 1 -c 1 -o gpurun_out/r01/prof_det_road1024 python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --nostats --variants det32 > gpurun_out/r01/ncu_det.log 2>&1
tail -2 gpurun_out/r01/ncu_det.log
