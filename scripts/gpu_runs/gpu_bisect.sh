cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/bis
for rep in 1 2; do
for c in 2860eea de1f1f3 168b378 649e4b2; do
  (cd abtest/$c && timeout 600 python scripts/diag.py --graph rmat:24 --roots 3 --reps 1 --nostats --variants default | sed "s/\"variant\": \"default\"/\"variant\": \"$c\"/" >> ../../gpurun_out/bis/diag.jsonl 2>> ../../gpurun_out/bis/err.log)
done
timeout 600 python scripts/diag.py --graph rmat:24 --roots 3 --reps 1 --nostats --variants default >> gpurun_out/bis/diag.jsonl 2>> gpurun_out/bis/err.log
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/bis/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -2 gpurun_out/bis/err.log
