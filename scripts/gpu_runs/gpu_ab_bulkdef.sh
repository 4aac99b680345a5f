cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/bd
for g in rmat:24 road:4900 rmat:22 grid:256 path:1e8 cat:20; do
  timeout 900 python scripts/diag.py --graph $g --roots 3 --reps 1 --nostats --variants default,bulk_copy,default,bulk_copy,default,bulk_copy >> gpurun_out/bd/diag.jsonl 2>> gpurun_out/bd/err.log
done
for k in 4 6 8; do
  timeout 900 python bench.py --config batch1024 --warmup 3 --concurrency $k > gpurun_out/bd/batch_k$k.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/bd/batch_k$k.json')); print('batch k=$k', d['value'], d['dfs_per_s'])"
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/bd/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -2 gpurun_out/bd/err.log
