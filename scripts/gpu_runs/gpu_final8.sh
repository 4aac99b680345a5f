cd $GRAFT_REPO_ROOT
O=gpurun_out/r01i_end
mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/gpu_tests_full.log 2>&1; echo "tests rc=$?" >> $O/gpu_tests_full.log
tail -3 $O/gpu_tests_full.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log; tail -2 $O/smoke.log
timeout 600 python bench.py > $O/bench_default.json 2> $O/bench_default.err
for c in rmat24; do
  timeout 900 python bench.py --config $c --steps 8 --warmup 3 --cpu-seconds 10 > $O/bench_$c.json 2> $O/bench_$c.err
done
for c in road24m rmat24; do
  f=$O/bench_$c.json; [ $c = road24m ] && f=$O/bench_default.json
  python -c "import json; d=json.load(open('$f')); print('$c', d['value'], d['ms_per_dfs'], 'cpu', d.get('cpu_baseline',{}).get('value'), 'e2e', d.get('e2e',{}).get('value'), 'roof', d['roofline']['frac'], 'clocks', d['clocks'])"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 2 -c 1 -o $O/prof_rmat24 python bench.py --config rmat24 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > $O/ncu_full_rmat.log 2>&1
ls $O
