# walker-kernel micro-optimisations (32-bit ring addresses in push/pop, one-ballot idle mask) vs HEAD
set -x
timeout 600 python -m pytest tests/test_gpu_walker.py -q -x --timeout 300 > gpurun_out/pytest_wmicro.log 2>&1; echo pytest rc=$?
tail -1 gpurun_out/pytest_wmicro.log
L="ab/head/libdfs.so paper_conf_ppopp_niul0c26_b200/libdfs.so"
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --batch 64 --reps 7 > gpurun_out/ab_wmicro_batch.jsonl 2>&1
grep -h lib gpurun_out/ab_wmicro_batch.jsonl || tail -5 gpurun_out/ab_wmicro_batch.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --config path100m --reps 3 --steps 2 > gpurun_out/ab_wmicro_path.jsonl 2>&1
grep -h lib gpurun_out/ab_wmicro_path.jsonl || tail -5 gpurun_out/ab_wmicro_path.jsonl
