# prefetch of the next stack entry's window after a pop (DFS_POPPF=1, ab/poppf) vs the default build
set -x
DFS_LIB=ab/poppf/libdfs.so timeout 600 python -m pytest tests/test_gpu_parity.py -q -x --timeout 300 > gpurun_out/pytest_poppf.log 2>&1; echo pytest rc=$?
tail -1 gpurun_out/pytest_poppf.log
L="paper_conf_ppopp_niul0c26_b200/libdfs.so ab/poppf/libdfs.so"
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --reps 7 --steps 8 > gpurun_out/ab_poppf_road24m.jsonl 2>&1
grep -h lib gpurun_out/ab_poppf_road24m.jsonl || tail -5 gpurun_out/ab_poppf_road24m.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --set deterministic=1 --config road24m --reps 1 --steps 1 --nroots 1 --validate 0 > gpurun_out/ab_poppf_det.jsonl 2>&1
grep -h lib gpurun_out/ab_poppf_det.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --config grid256 --reps 5 --steps 6 > gpurun_out/ab_poppf_grid256.jsonl 2>&1
grep -h lib gpurun_out/ab_poppf_grid256.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --config caterpillar --reps 3 --steps 2 > gpurun_out/ab_poppf_caterpillar.jsonl 2>&1
grep -h lib gpurun_out/ab_poppf_caterpillar.jsonl
