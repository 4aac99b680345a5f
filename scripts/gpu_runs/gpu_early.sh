cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/early
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubench_chain scripts/ubench_chain.cu && timeout 60 /tmp/ubench_chain > gpurun_out/early/ubench_chain.json 2>&1
cat gpurun_out/early/ubench_chain.json
for gspec in grid:256 cat:20 road:4900 path:1e8; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 2 --nostats --variants default,early,default,early >> gpurun_out/early/ab.jsonl 2>> gpurun_out/early/ab.err
  timeout 900 python scripts/diag.py --graph $gspec --roots 1 --reps 1 --variants w0det,w0detearly,w0,w0early >> gpurun_out/early/stats.jsonl 2>> gpurun_out/early/ab.err
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/early/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in d.items(): print(k, 'mean ms', round(sum(v)/len(v),3), v)
for l in open('gpurun_out/early/stats.jsonl'):
    r=json.loads(l); print(r['graph'], r['variant'], r['ms'], r['cyc_per_window'], r['windows_per_claim'])
PY
tail -3 gpurun_out/early/ab.err
