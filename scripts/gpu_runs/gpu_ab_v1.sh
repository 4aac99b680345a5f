# A/B of the 32-wide step shape: working tree vs abtest/base on chain-bound graphs
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/v1b
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/v1b/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/v1b/parity.log
tail -2 gpurun_out/v1b/parity.log
for gspec in path:1e8 grid:256 road:4900; do
  for rep in 1 2; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default >> gpurun_out/v1b/ab.jsonl 2>> gpurun_out/v1b/ab.err
  (cd abtest/base && timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "base"/' >> ../../gpurun_out/v1b/ab.jsonl 2>> ../../gpurun_out/v1b/ab.err)
  done
done
timeout 900 python scripts/diag.py --graph path:1e6 --roots 1 --reps 1 --nostats --variants det >> gpurun_out/v1b/ab.jsonl 2>> gpurun_out/v1b/ab.err
(cd abtest/base && timeout 900 python scripts/diag.py --graph path:1e6 --roots 1 --reps 1 --nostats --variants det | sed 's/"variant": "det"/"variant": "base-det"/' >> ../../gpurun_out/v1b/ab.jsonl 2>> ../../gpurun_out/v1b/ab.err)
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/v1b/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
