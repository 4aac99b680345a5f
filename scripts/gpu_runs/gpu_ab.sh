cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab
for h in b476c53 bf06468 acabee7 de4f2df; do
  for c in caterpillar path100m road24m; do
    (cd abtest/$h && timeout 900 python bench.py --config $c --steps 4 --warmup 2 --no-e2e --no-cpu-baseline --no-validate > ../../gpurun_out/ab/${h}_$c.json 2>/dev/null)
    python -c "import json; d=json.load(open('gpurun_out/ab/${h}_$c.json')); print('$h', '$c', d['value'], d['ms_per_dfs'])" || echo "$h $c failed"
  done
done
