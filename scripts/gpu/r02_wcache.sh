# hub-window cache (DFS_WCACHE=1 build in ab/wcache): parity with that build, then A/B vs the default
export DFS_SKIP_FULLSIZE=0
DFS_LIB=ab/wcache/libdfs.so timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_capi_batch.py "tests/test_gpu_fullsize.py::test_full_configs_valid" -q -x --timeout 300 -rf > gpurun_out/pytest_wcache.log 2>&1; echo wcache tests rc=$?
tail -4 gpurun_out/pytest_wcache.log
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/wcache/libdfs.so --config rmat24 --reps 5 --steps 6 > gpurun_out/ab_wcache_rmat.jsonl 2>&1
grep lib gpurun_out/ab_wcache_rmat.jsonl || tail -20 gpurun_out/ab_wcache_rmat.jsonl
timeout 600 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/wcache/libdfs.so --config road24m --reps 3 --steps 6 > gpurun_out/ab_wcache_road.jsonl 2>&1
grep lib gpurun_out/ab_wcache_road.jsonl || tail -20 gpurun_out/ab_wcache_road.jsonl
DFS_LIB=ab/wcache/libdfs.so timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:dfs_persistent_kernel --launch-skip 1 -c 1 --csv \
  python scripts/ncu_run.py --config rmat24 > gpurun_out/ncu_wcache_rmat.csv 2>&1; echo ncu rc=$?
grep -E "dram__bytes|gpu__time" gpurun_out/ncu_wcache_rmat.csv | cut -c1-300
