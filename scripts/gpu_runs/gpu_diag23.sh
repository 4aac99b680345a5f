cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python scripts/diag.py --graph rmat:22 --roots 3 --reps 2 --nostats --timeline 5 --variants default,w32,w128 > gpurun_out/diag23.jsonl 2> gpurun_out/diag23.err
timeout 900 python bench.py --config rmat24 --steps 4 --warmup 2 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/b23_rmat128.json 2>/dev/null
python - <<'PY'
import json, collections
agg = collections.defaultdict(list)
for l in open('gpurun_out/diag23.jsonl'):
    d=json.loads(l); agg[d['graph']+' '+d['variant']].append(d['ms']); print(d['graph'], d['variant'], d['root'], d['ms'], d.get('busy_by_5pct'))
for k,v in agg.items(): print('MEAN', k, round(sum(v)/len(v),2))
d=json.load(open('gpurun_out/b23_rmat128.json')); print('rmat24 bench', d['value'], d['ms_per_dfs'])
PY
