# why was the edge-annotated adjacency neutral? single-warp step latency (deterministic mode) and
# ncu source-level stalls of the ADJ build vs the default build on road24m root 0
set -x
L="paper_conf_ppopp_niul0c26_b200/libdfs.so ab/adj/libdfs.so"
timeout 900 python scripts/ab_libs.py --libs $L --set deterministic=1 --config road24m --reps 1 --steps 1 --nroots 1 --validate 0 > gpurun_out/ab_adj_det.jsonl 2>&1
grep -h lib gpurun_out/ab_adj_det.jsonl || tail -5 gpurun_out/ab_adj_det.jsonl
mkdir -p /tmp/prof
timeout 900 env DFS_LIB=ab/adj/libdfs.so ncu --set full --import-source on --clock-control none -k regex:dfs_persistent_kernel --launch-skip 1 -c 1 \
  -o /tmp/prof/adj python scripts/ncu_run.py --config road24m > gpurun_out/prof_adj.log 2>&1; echo ncu rc=$?
ncu -i /tmp/prof/adj.ncu-rep --page raw --csv > gpurun_out/prof_adj_raw.csv 2>/dev/null
ncu -i /tmp/prof/adj.ncu-rep --page source --csv > gpurun_out/prof_adj_source.csv 2>/dev/null
gzip -9 gpurun_out/prof_adj_source.csv
