cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab2
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/ab2/tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/ab2/tests.log; tail -2 gpurun_out/ab2/tests.log
for c in caterpillar path100m road24m rmat24; do
  timeout 900 python bench.py --config $c --steps 4 --warmup 2 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/ab2/new_$c.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/ab2/new_$c.json')); print('new', '$c', d['value'], d['ms_per_dfs'])" || echo "new $c failed"
  (cd abtest/b476c53 && timeout 900 python bench.py --config $c --steps 4 --warmup 2 --no-e2e --no-cpu-baseline --no-validate > ../../gpurun_out/ab2/old_$c.json 2>/dev/null)
  python -c "import json; d=json.load(open('gpurun_out/ab2/old_$c.json')); print('old', '$c', d['value'], d['ms_per_dfs'])" || echo "old $c failed"
done
