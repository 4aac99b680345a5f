# edge-annotated adjacency for the 32-wide step (default build) vs col_idx + row_ptr (ab/noadj)
set -x
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stack_script.py -q -x --timeout 600 > gpurun_out/pytest_adj.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_adj.log
for c in road24m grid256; do
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/noadj/libdfs.so --config $c --reps 5 --steps 8 > gpurun_out/ab_adj_$c.jsonl 2>&1
grep -h lib gpurun_out/ab_adj_$c.jsonl || tail -5 gpurun_out/ab_adj_$c.jsonl
done
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/noadj/libdfs.so --config caterpillar --reps 3 --steps 2 > gpurun_out/ab_adj_caterpillar.jsonl 2>&1
grep -h lib gpurun_out/ab_adj_caterpillar.jsonl
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/noadj/libdfs.so --config path100m --set walker_lanes=32 --reps 3 --steps 2 > gpurun_out/ab_adj_path32.jsonl 2>&1
grep -h lib gpurun_out/ab_adj_path32.jsonl
