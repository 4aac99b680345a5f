# A/B of speculation bits on the lean step
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/spec
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/spec/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/spec/parity.log
tail -2 gpurun_out/spec/parity.log
for gspec in grid:256 road:4900 path:1e8 rmat:22; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default,early,specpop,specboth,default,early,specpop,specboth >> gpurun_out/spec/ab.jsonl 2>> gpurun_out/spec/ab.err
done
timeout 900 python scripts/diag.py --graph rmat:22 --roots 3 --reps 1 --nostats --variants default,specpop128,default,specpop128 >> gpurun_out/spec/ab.jsonl 2>> gpurun_out/spec/ab.err
timeout 900 python scripts/diag.py --graph cat:20 --roots 1 --reps 1 --nostats --variants default,early,specpop,specboth >> gpurun_out/spec/ab.jsonl 2>> gpurun_out/spec/ab.err
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/spec/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -3 gpurun_out/spec/ab.err
