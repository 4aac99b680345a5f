cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/rm24
for rep in 1 2; do
for c in rmat24 road24m; do
  timeout 900 python bench.py --config $c --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/rm24/head_${c}_$rep.json 2>/dev/null
  (cd abtest/base && timeout 900 python bench.py --config $c --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > ../../gpurun_out/rm24/base_${c}_$rep.json 2>/dev/null)
done
done
timeout 600 python scripts/diag.py --graph rmat:24 --roots 3 --reps 1 --nostats --variants default,st1,noearly >> gpurun_out/rm24/diag.jsonl 2>> gpurun_out/rm24/err.log
(cd abtest/base && timeout 600 python scripts/diag.py --graph rmat:24 --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "base"/' >> ../../gpurun_out/rm24/diag.jsonl 2>> ../../gpurun_out/rm24/err.log)
for f in gpurun_out/rm24/*.json; do python -c "import json,sys; d=json.load(open('$f')); print('$f', d['value'], d['ms_per_dfs'], d['ms_per_dfs_median'])"; done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/rm24/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
