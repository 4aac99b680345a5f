cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/lw
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/lw/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/lw/parity.log
tail -3 gpurun_out/lw/parity.log
for g in rmat:24 rmat:22 road:4900; do
for rep in 1 2; do
  (cd abtest/base && timeout 600 python scripts/diag.py --graph $g --roots 3 --reps 1 --nostats --variants default | sed "s/\"variant\": \"default\"/\"variant\": \"base\"/" >> ../../gpurun_out/lw/diag.jsonl 2>> ../../gpurun_out/lw/err.log)
  timeout 600 python scripts/diag.py --graph $g --roots 3 --reps 1 --nostats --variants default >> gpurun_out/lw/diag.jsonl 2>> gpurun_out/lw/err.log
done
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/lw/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -2 gpurun_out/lw/err.log
