# round-2 session-2 end check of the committed build: smoke, all GPU tests, default bench
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_end.log 2>&1; echo smoke rc=$?
tail -1 gpurun_out/smoke_end.log
timeout 1500 python -m pytest tests -m gpu -q -rf --timeout 600 --durations=5 > gpurun_out/pytest_gpu_end.log 2>&1; echo pytest rc=$?
tail -2 gpurun_out/pytest_gpu_end.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_end.json 2> gpurun_out/bench_end.err; echo bench rc=$?
tail -2 gpurun_out/bench_end.err
