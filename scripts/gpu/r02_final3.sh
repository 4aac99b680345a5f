# round-2 pass 3 (final defaults): all GPU tests + smoke, bench, launch lists, ncu --set full captures
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 1800 python -m pytest tests -m gpu -q -rf --timeout 600 --durations=10 > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -4 gpurun_out/pytest_gpu.log
timeout 1200 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_road24m.csv \
  python bench.py --steps 3 --warmup 3 --no-batch --no-rmat --no-e2e --no-cpu-baseline --no-validate > /dev/null 2>&1; echo launches road rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_batch.csv \
  python bench.py --config batch1024 --batch-roots 64 --warmup 3 --no-cpu-baseline --no-validate --no-e2e > /dev/null 2>&1; echo launches batch rc=$?
mkdir -p /tmp/prof
prof() {  # name kernel-regex skip args...
  local name=$1 k=$2 skip=$3; shift 3
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:$k --launch-skip $skip -c 1 \
    -o /tmp/prof/$name python scripts/ncu_run.py "$@" > gpurun_out/prof_$name.log 2>&1; echo ncu $name rc=$?
  ncu -i /tmp/prof/$name.ncu-rep --page raw --csv > gpurun_out/prof_${name}_raw.csv 2>/dev/null
  ncu -i /tmp/prof/$name.ncu-rep --page source --csv > gpurun_out/prof_${name}_source.csv 2>/dev/null
  gzip -9 gpurun_out/prof_${name}_source.csv
}
prof road24m dfs_persistent_kernel 1 --config road24m
prof rmat24 dfs_persistent_kernel 1 --config rmat24
prof path100m dfs_walker_kernel 1 --config path100m
prof batch dfs_walker_kernel 8 --config road24m --batch 8
cp /tmp/prof/road24m.ncu-rep gpurun_out/prof_road24m.ncu-rep
du -sh gpurun_out
