cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/nb
for g in rmat:24 rmat:22 road:4900; do
for rep in 1 2; do
  for v in 168b378 nb pm nbpm; do
  (cd abtest/$v && timeout 600 python scripts/diag.py --graph $g --roots 3 --reps 1 --nostats --variants default | sed "s/\"variant\": \"default\"/\"variant\": \"$v\"/" >> ../../gpurun_out/nb/diag.jsonl 2>> ../../gpurun_out/nb/err.log)
  done
  timeout 600 python scripts/diag.py --graph $g --roots 3 --reps 1 --nostats --variants default >> gpurun_out/nb/diag.jsonl 2>> gpurun_out/nb/err.log
done
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/nb/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -2 gpurun_out/nb/err.log
