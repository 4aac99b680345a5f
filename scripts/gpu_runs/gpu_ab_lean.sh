# A/B: working tree (lean 32-wide step) vs abtest/base (HEAD) on the chain-bound graphs
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/lean
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/lean/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/lean/parity.log
tail -3 gpurun_out/lean/parity.log
for gspec in grid:256 road:4900 path:1e8 cat:20; do
  for rep in 1 2; do
    timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "lean"/' >> gpurun_out/lean/ab.jsonl 2>> gpurun_out/lean/ab.err
    (cd abtest/base && timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "base"/' >> ../../gpurun_out/lean/ab.jsonl 2>> ../../gpurun_out/lean/ab.err)
  done
done
timeout 900 python scripts/diag.py --graph path:1e6 --roots 1 --reps 1 --nostats --variants det | sed 's/"variant": "det"/"variant": "lean-det"/' >> gpurun_out/lean/ab.jsonl 2>> gpurun_out/lean/ab.err
(cd abtest/base && timeout 900 python scripts/diag.py --graph path:1e6 --roots 1 --reps 1 --nostats --variants det | sed 's/"variant": "det"/"variant": "base-det"/' >> ../../gpurun_out/lean/ab.jsonl 2>> ../../gpurun_out/lean/ab.err)
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/lean/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -3 gpurun_out/lean/ab.err
