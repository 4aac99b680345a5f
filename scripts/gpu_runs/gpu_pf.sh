cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/pf
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubench_chain scripts/ubench_chain.cu && timeout 120 /tmp/ubench_chain > gpurun_out/pf/ubench_chain.json 2>&1
cat gpurun_out/pf/ubench_chain.json
for gspec in grid:256 road:4900 path:1e8 cat:20; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default,pf2,pf4,pf8,default,pf4 >> gpurun_out/pf/ab.jsonl 2>> gpurun_out/pf/ab.err
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/pf/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in d.items(): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -3 gpurun_out/pf/ab.err
