cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/cl2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/cl2/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "cluster or stress or deterministic" > gpurun_out/cl2/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/cl2/parity.log
tail -3 gpurun_out/cl2/parity.log
for gspec in road:4900 rmat:22 path:1e8; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default,cl1,cl2,cl2late,early2,default,cl1,cl2,cl2late,early2 >> gpurun_out/cl2/ab.jsonl 2>> gpurun_out/cl2/ab.err
done
timeout 300 python scripts/diag.py --graph path:1e6 --roots 1 --reps 3 --nostats --variants det,detearly,det,detearly >> gpurun_out/cl2/ab.jsonl 2>> gpurun_out/cl2/ab.err
timeout 300 python scripts/diag.py --graph cat:20 --roots 1 --reps 1 --nostats --variants default,early2,cl2late >> gpurun_out/cl2/ab.jsonl 2>> gpurun_out/cl2/ab.err
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/cl2/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -3 gpurun_out/cl2/ab.err
