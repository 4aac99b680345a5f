cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/bulk2
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/bulk2/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/bulk2/parity.log
tail -2 gpurun_out/bulk2/parity.log
for gspec in rmat:22 road:4900 cat:20 grid:256 path:1e8; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default,bulk,default,bulk >> gpurun_out/bulk2/ab.jsonl 2>> gpurun_out/bulk2/ab.err
  (cd abtest/base && timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "base"/' >> ../../gpurun_out/bulk2/ab.jsonl 2>> ../../gpurun_out/bulk2/ab.err)
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/bulk2/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -3 gpurun_out/bulk2/ab.err
