cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r01b
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider > gpurun_out/r01b/gpu_tests_full.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01b/gpu_tests_full.log
tail -3 gpurun_out/r01b/gpu_tests_full.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01b/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r01b/smoke.log; tail -2 gpurun_out/r01b/smoke.log
for c in road24m grid256 rmat24 path100m caterpillar; do
  timeout 900 python bench.py --config $c --steps 8 --warmup 3 --cpu-seconds 10 > gpurun_out/r01b/bench_$c.json 2> gpurun_out/r01b/bench_$c.err
  python -c "import json; d=json.load(open('gpurun_out/r01b/bench_$c.json')); print('$c', d['value'], d['ms_per_dfs'], 'cpu', d.get('cpu_baseline',{}).get('value'), 'e2e', d.get('e2e',{}).get('value'), 'roof', d['roofline']['frac'], 'traffic', d['roofline']['traffic'])" || tail -3 gpurun_out/r01b/bench_$c.err
done
timeout 900 python bench.py --config batch1024 --warmup 3 > gpurun_out/r01b/bench_batch1024.json 2> gpurun_out/r01b/bench_batch1024.err
python -c "import json; d=json.load(open('gpurun_out/r01b/bench_batch1024.json')); print('batch1024', d['value'], d['dfs_per_s'], d['concurrency'])"
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r01b/bench_reference.json 2> gpurun_out/r01b/bench_reference.err; head -c 300 gpurun_out/r01b/bench_reference.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01b/launches_road24m.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/r01b/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 2 -c 1 -o gpurun_out/r01b/prof_road24m python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/r01b/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 2 -c 1 -o gpurun_out/r01b/prof_rmat24 python bench.py --config rmat24 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/r01b/ncu_full_rmat.log 2>&1
ls gpurun_out/r01b
