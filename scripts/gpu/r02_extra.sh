# batch slots on all 148 SMs (default) vs 8 x 18 blocks (ab/noextra)
timeout 1500 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/noextra/libdfs.so --config road24m --reps 3 --batch 128 > gpurun_out/ab_extra_batch.jsonl 2>&1
grep lib gpurun_out/ab_extra_batch.jsonl || tail -20 gpurun_out/ab_extra_batch.jsonl
timeout 900 python -m pytest tests/test_gpu_capi_batch.py tests/test_gpu_parity.py tests/test_gpu_walker.py -q -x --timeout 300 -k "batch or concurrent or host" > gpurun_out/pytest_extra.log 2>&1; echo tests rc=$?
tail -3 gpurun_out/pytest_extra.log
