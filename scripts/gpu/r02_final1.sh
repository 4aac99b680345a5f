# round-2 pass 1: all GPU tests + smoke, bench, launch lists, ncu --set full captures
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 1800 python -m pytest tests -m gpu -q -rf --timeout 600 --durations=10 > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -15 gpurun_out/pytest_gpu.log
timeout 1200 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
# launch lists (cold-cache, serialised: shares, not absolutes)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_road24m.csv \
  python bench.py --steps 3 --warmup 3 --no-batch --no-rmat --no-e2e --no-cpu-baseline --no-validate > /dev/null 2>&1; echo launches road rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_batch.csv \
  python bench.py --config batch1024 --batch-roots 64 --warmup 3 --no-cpu-baseline --no-validate > /dev/null 2>&1; echo launches batch rc=$?
# top kernels, --set full (one launch each after a warm-up)
timeout 900 ncu --set full --import-source on --clock-control none -k regex:dfs_persistent_kernel --launch-skip 1 -c 1 \
  -o gpurun_out/prof_road24m python scripts/ncu_run.py --config road24m > gpurun_out/prof_road24m.log 2>&1; echo ncu road rc=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:dfs_persistent_kernel --launch-skip 1 -c 1 \
  -o gpurun_out/prof_rmat24 python scripts/ncu_run.py --config rmat24 > gpurun_out/prof_rmat24.log 2>&1; echo ncu rmat rc=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:dfs_walker_kernel --launch-skip 1 -c 1 \
  -o gpurun_out/prof_path100m python scripts/ncu_run.py --config path100m > gpurun_out/prof_path100m.log 2>&1; echo ncu path rc=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:dfs_walker_kernel --launch-skip 8 -c 1 \
  -o gpurun_out/prof_batch python scripts/ncu_run.py --config road24m --batch 8 > gpurun_out/prof_batch.log 2>&1; echo ncu batch rc=$?
ls -la gpurun_out
