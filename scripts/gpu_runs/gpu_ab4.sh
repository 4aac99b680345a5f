cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab4
for c in road24m caterpillar path100m rmat24; do
  timeout 900 python bench.py --config $c --steps 6 --warmup 2 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/ab4/r256_$c.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/ab4/r256_$c.json')); print('ring256', '$c', d['value'], d['ms_per_dfs'])" || echo "256 $c failed"
  for v in ring128 ring64; do
    (cd abtest/$v && timeout 900 python bench.py --config $c --steps 6 --warmup 2 --no-e2e --no-cpu-baseline --no-validate > ../../gpurun_out/ab4/${v}_$c.json 2>/dev/null)
    python -c "import json; d=json.load(open('gpurun_out/ab4/${v}_$c.json')); print('$v', '$c', d['value'], d['ms_per_dfs'])" || echo "$v $c failed"
  done
done
