# lazy probes (skip the window's probes when the speculative claim wins), alone and with the
# edge-annotated adjacency, vs the session-start build (ab/head)
set -x
L="ab/head/libdfs.so ab/lazy/libdfs.so ab/adjlazy/libdfs.so"
for lib in ab/lazy/libdfs.so ab/adjlazy/libdfs.so; do
DFS_LIB=$lib timeout 600 python -m pytest tests/test_gpu_parity.py -q -x --timeout 300 -k "deterministic or valid or stress" > gpurun_out/pytest_$(basename $(dirname $lib)).log 2>&1; echo pytest $lib rc=$?
tail -2 gpurun_out/pytest_$(basename $(dirname $lib)).log
done
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --reps 5 --steps 8 > gpurun_out/ab_lazy_road24m.jsonl 2>&1
grep -h lib gpurun_out/ab_lazy_road24m.jsonl || tail -5 gpurun_out/ab_lazy_road24m.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --set deterministic=1 --config road24m --reps 1 --steps 1 --nroots 1 --validate 0 > gpurun_out/ab_lazy_det.jsonl 2>&1
grep -h lib gpurun_out/ab_lazy_det.jsonl || tail -5 gpurun_out/ab_lazy_det.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --config grid256 --reps 5 --steps 6 > gpurun_out/ab_lazy_grid256.jsonl 2>&1
grep -h lib gpurun_out/ab_lazy_grid256.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --config caterpillar --reps 3 --steps 2 > gpurun_out/ab_lazy_caterpillar.jsonl 2>&1
grep -h lib gpurun_out/ab_lazy_caterpillar.jsonl
