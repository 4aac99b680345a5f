# 128-wide step: row_ptr prefetch width for candidate lanes (DFS_PF_LANES128 = 2 default, 1, 0)
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/pf1/libdfs.so ab/pf0/libdfs.so --config rmat24 --reps 5 --steps 6 > gpurun_out/ab_pf_rmat.jsonl 2>&1
grep lib gpurun_out/ab_pf_rmat.jsonl || tail -20 gpurun_out/ab_pf_rmat.jsonl
for v in pf1 pf0; do
DFS_LIB=ab/$v/libdfs.so timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_op_read.sum --clock-control none -k regex:dfs_persistent_kernel --launch-skip 1 -c 1 --csv \
  python scripts/ncu_run.py --config rmat24 > gpurun_out/ncu_${v}_rmat.csv 2>&1; echo ncu $v rc=$?
grep -E "dram__bytes|gpu__time|lts__t_sectors" gpurun_out/ncu_${v}_rmat.csv | awk -F'","' '{print $13, $15}'
done
