cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/prof4
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 1 -c 1 -o gpurun_out/prof4/det_path1e6 python scripts/diag.py --graph path:1e6 --roots 1 --reps 1 --nostats --variants det > gpurun_out/prof4/ncu_det_path.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 1 -c 1 -o gpurun_out/prof4/par_road4900 python scripts/diag.py --graph road:4900 --roots 1 --reps 1 --nostats --variants default > gpurun_out/prof4/ncu_par_road.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 1 -c 1 -o gpurun_out/prof4/par_cat20 python scripts/diag.py --graph cat:20 --roots 1 --reps 1 --nostats --variants default > gpurun_out/prof4/ncu_par_cat.log 2>&1
tail -2 gpurun_out/prof4/*.log
ls -la gpurun_out/prof4
