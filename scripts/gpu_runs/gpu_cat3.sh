cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/cat3
timeout 900 python scripts/diag.py --graph cat:20 --roots 2 --reps 1 --nostats --variants default,nointra,b16,b32,b74,w8 >> gpurun_out/cat3/diag.jsonl 2>> gpurun_out/cat3/err.log
timeout 600 python scripts/diag.py --graph path:1e6 --roots 1 --reps 2 --nostats --variants det >> gpurun_out/cat3/diag.jsonl 2>> gpurun_out/cat3/err.log
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/cat3/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
