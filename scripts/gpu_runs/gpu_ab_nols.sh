cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/nols
for gspec in path:1e8 grid:256; do
  for rep in 1 2; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default >> gpurun_out/nols/ab.jsonl 2>> gpurun_out/nols/ab.err
  (cd abtest/base && timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "base"/' >> ../../gpurun_out/nols/ab.jsonl 2>> ../../gpurun_out/nols/ab.err)
  (cd abtest/nols && timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "nols"/' >> ../../gpurun_out/nols/ab.jsonl 2>> ../../gpurun_out/nols/ab.err)
  done
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/nols/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
