set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 1500 python -m pytest tests -m gpu -q -rf --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -30 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -5 gpurun_out/bench.err
timeout 600 python scripts/ab_libs.py --libs ab/r01/libdfs.so paper_conf_ppopp_niul0c26_b200/libdfs.so --config road24m --reps 5 --steps 8 > gpurun_out/ab_road.jsonl 2>&1
timeout 600 python scripts/ab_libs.py --libs ab/r01/libdfs.so paper_conf_ppopp_niul0c26_b200/libdfs.so --config rmat24 --reps 5 --steps 8 > gpurun_out/ab_rmat.jsonl 2>&1
cat gpurun_out/ab_road.jsonl gpurun_out/ab_rmat.jsonl | grep lib
