# warp-kernel donation (block mailboxes) vs donate=0 vs the previous build (ab/noadj = HEAD code)
set -x
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stack_script.py -q -x --timeout 300 > gpurun_out/pytest_don.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_don.log
L="paper_conf_ppopp_niul0c26_b200/libdfs.so ab/noadj/libdfs.so"
timeout 900 python scripts/ab_libs.py --libs $L --variant "" --variant donate=0 --config road24m --reps 5 --steps 8 > gpurun_out/ab_don_road24m.jsonl 2>&1
grep -h lib gpurun_out/ab_don_road24m.jsonl || tail -5 gpurun_out/ab_don_road24m.jsonl
for c in grid256 rmat24; do
timeout 900 python scripts/ab_libs.py --libs $L --config $c --reps 5 --steps 6 > gpurun_out/ab_don_$c.jsonl 2>&1
grep -h lib gpurun_out/ab_don_$c.jsonl || tail -5 gpurun_out/ab_don_$c.jsonl
done
timeout 900 python scripts/ab_libs.py --libs $L --config caterpillar --reps 3 --steps 2 > gpurun_out/ab_don_caterpillar.jsonl 2>&1
grep -h lib gpurun_out/ab_don_caterpillar.jsonl
