# RMAT-24 after the row_ptr-prefetch change: next-window L1 prefetch (ab/nwpf0), persisting L2, window width
timeout 1200 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/nwpf0/libdfs.so --config rmat24 --reps 5 --steps 6 \
  --variant "" --variant "l2_persist_mb=-1" --variant "window=32" --variant "speculate=1" > gpurun_out/ab_rmat2.jsonl 2>&1
grep lib gpurun_out/ab_rmat2.jsonl || tail -20 gpurun_out/ab_rmat2.jsonl
DFS_LIB=ab/nwpf0/libdfs.so timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:dfs_persistent_kernel --launch-skip 1 -c 1 --csv \
  python scripts/ncu_run.py --config rmat24 > gpurun_out/ncu_nwpf0_rmat.csv 2>&1; echo ncu rc=$?
grep -E "dram__bytes|gpu__time" gpurun_out/ncu_nwpf0_rmat.csv | awk -F'","' '{print $13, $15}'
