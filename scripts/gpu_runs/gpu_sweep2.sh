cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/sw2
for g in road:4900 rmat:24; do
for rep in 1 2; do
  timeout 900 python scripts/diag.py --graph $g --roots 3 --reps 1 --nostats --variants default,h2c1,h1c4,si64,si256,si8,pb2,bmin64,bmax1k,bmax4k >> gpurun_out/sw2/diag.jsonl 2>> gpurun_out/sw2/err.log
done
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/sw2/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -2 gpurun_out/sw2/err.log
