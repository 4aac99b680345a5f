# windowed Alg 3 victim scan in the walker kernel (default build) vs the full CTA scan (ab/fullscan)
timeout 1500 python -m pytest tests/test_gpu_walker.py tests/test_gpu_stack_script.py -q -x --timeout 150 -rf > gpurun_out/pytest_scan.log 2>&1; echo walker tests rc=$?
tail -3 gpurun_out/pytest_scan.log
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/fullscan/libdfs.so --config road24m --reps 3 --batch 64 \
  --variant "" --variant "steal_period=4" --variant "steal_period=64" > gpurun_out/ab_scan_batch.jsonl 2>&1
grep lib gpurun_out/ab_scan_batch.jsonl || tail -20 gpurun_out/ab_scan_batch.jsonl
timeout 600 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/fullscan/libdfs.so --config path100m --reps 3 --steps 4 > gpurun_out/ab_scan_path.jsonl 2>&1
grep lib gpurun_out/ab_scan_path.jsonl || tail -20 gpurun_out/ab_scan_path.jsonl
