cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/bulk
for gspec in rmat:22 road:4900 cat:20 grid:256 path:1e8; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default,bulk,w16,bulkw16,default,bulk >> gpurun_out/bulk/ab.jsonl 2>> gpurun_out/bulk/ab.err
done
timeout 900 python scripts/diag.py --graph rmat:22 --roots 1 --reps 1 --timeline 5 --variants bulk >> gpurun_out/bulk/tl.jsonl 2>> gpurun_out/bulk/ab.err
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/bulk/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
for l in open('gpurun_out/bulk/tl.jsonl'):
    r=json.loads(l); print(r['ms'], r['claims'], r['claims_by_5pct'])
PY
tail -3 gpurun_out/bulk/ab.err
