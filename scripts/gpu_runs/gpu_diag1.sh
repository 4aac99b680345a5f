cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python scripts/diag.py --graph road:4900 --roots 2 --variants default,w16,w8,hot16,hot8,cold32,h8c16,random,nointer,nointra,b74 > gpurun_out/diag_road.jsonl 2> gpurun_out/diag_road.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 2 --variants default,w16,hot8,h8c16,nointer > gpurun_out/diag_rmat.jsonl 2> gpurun_out/diag_rmat.err
timeout 300 python scripts/diag.py --graph grid:256 --roots 1 --variants default,w8,det > gpurun_out/diag_grid.jsonl 2>> gpurun_out/diag_rmat.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 1 -c 1 -o gpurun_out/prof_road python scripts/diag.py --graph road:4900 --roots 1 --reps 1 > gpurun_out/ncu_full.log 2>&1
cat gpurun_out/diag_road.jsonl gpurun_out/diag_rmat.jsonl gpurun_out/diag_grid.jsonl; tail -3 gpurun_out/diag_road.err gpurun_out/ncu_full.log
