# runtime-parameter sweep of the rebuilt 128-wide kernel on RMAT-24 (no code change)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/sweep
timeout 1200 python scripts/diag.py --graph rmat:24 --roots 3 --reps 1 --nostats --variants default,l2off,l2p96,h2c1,h4c4,sp16,sp64,st4,nohalf,default,l2off,l2p96,h2c1,h4c4,sp16,sp64,st4,nohalf > gpurun_out/sweep/rmat24.jsonl 2> gpurun_out/sweep/err.log
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/sweep/rmat24.jsonl'):
    r=json.loads(l); d[r['variant']].append(r['ms'])
base=sum(d['default'])/len(d['default'])
for k,v in sorted(d.items(), key=lambda kv: sum(kv[1])/len(kv[1])): print(k, 'mean ms', round(sum(v)/len(v),3), 'vs default', round(sum(v)/len(v)/base,3))
PY
tail -2 gpurun_out/sweep/err.log
