cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
free -g > gpurun_out/host_mem.txt; nproc >> gpurun_out/host_mem.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider --durations=15 > gpurun_out/gpu_tests_full.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests_full.log
tail -25 gpurun_out/gpu_tests_full.log
for c in road24m grid256 rmat24 path100m caterpillar; do
  timeout 900 python bench.py --config $c --steps 6 --warmup 3 --no-e2e --cpu-seconds 8 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo "$c rc=$?"
  cat gpurun_out/bench_$c.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'], d['value'], d['unit'], d['ms_per_dfs'], 'cpu', d.get('cpu_baseline',{}).get('value'), 'roof', d['roofline']['frac'])" 2>/dev/null
done
