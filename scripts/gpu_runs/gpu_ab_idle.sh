cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/idle
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "stress or fault" > gpurun_out/idle/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/idle/parity.log
tail -3 gpurun_out/idle/parity.log
for gspec in road:4900 rmat:22 grid:256 path:1e8; do
  for rep in 1 2 3; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default >> gpurun_out/idle/ab.jsonl 2>> gpurun_out/idle/ab.err
  (cd abtest/base && timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "base"/' >> ../../gpurun_out/idle/ab.jsonl 2>> ../../gpurun_out/idle/ab.err)
  done
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/idle/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -3 gpurun_out/idle/ab.err
