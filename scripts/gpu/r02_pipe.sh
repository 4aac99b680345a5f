# pipelined claim in the 32-wide step (default build) vs DFS_PIPE=0 (ab/nopipe) vs the previous build (ab/head)
set -x
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stack_script.py -q -x --timeout 300 > gpurun_out/pytest_pipe.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_pipe.log
L="paper_conf_ppopp_niul0c26_b200/libdfs.so ab/nopipe/libdfs.so ab/head/libdfs.so"
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --reps 5 --steps 8 > gpurun_out/ab_pipe_road24m.jsonl 2>&1
grep -h lib gpurun_out/ab_pipe_road24m.jsonl || tail -5 gpurun_out/ab_pipe_road24m.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --set deterministic=1 --config road24m --reps 1 --steps 1 --nroots 1 --validate 0 > gpurun_out/ab_pipe_det.jsonl 2>&1
grep -h lib gpurun_out/ab_pipe_det.jsonl || tail -5 gpurun_out/ab_pipe_det.jsonl
for c in grid256 rmat24; do
timeout 900 python scripts/ab_libs.py --libs $L --config $c --reps 5 --steps 6 > gpurun_out/ab_pipe_$c.jsonl 2>&1
grep -h lib gpurun_out/ab_pipe_$c.jsonl || tail -5 gpurun_out/ab_pipe_$c.jsonl
done
timeout 900 python scripts/ab_libs.py --libs $L --config caterpillar --reps 3 --steps 2 > gpurun_out/ab_pipe_caterpillar.jsonl 2>&1
grep -h lib gpurun_out/ab_pipe_caterpillar.jsonl
