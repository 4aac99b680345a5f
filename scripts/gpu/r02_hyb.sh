# DFS_HYB: 32-wide step for short lists inside the 128-wide kernel, vs the session-start build
set -x
DFS_LIB=ab/hyb/libdfs.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x --timeout 600 -k "rmat or 128 or window or deterministic or stress or valid" > gpurun_out/pytest_hyb.log 2>&1; echo pytest rc=$?
tail -2 gpurun_out/pytest_hyb.log
L="ab/head/libdfs.so ab/hyb/libdfs.so paper_conf_ppopp_niul0c26_b200/libdfs.so"
timeout 900 python scripts/ab_libs.py --libs $L --config rmat24 --reps 7 --steps 6 > gpurun_out/ab_hyb_rmat24.jsonl 2>&1
grep -h lib gpurun_out/ab_hyb_rmat24.jsonl || tail -5 gpurun_out/ab_hyb_rmat24.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --set window=128 --reps 3 --steps 4 > gpurun_out/ab_hyb_road128.jsonl 2>&1
grep -h lib gpurun_out/ab_hyb_road128.jsonl || tail -5 gpurun_out/ab_hyb_road128.jsonl
