# A/B: unified lean step + leaf skip (working tree) vs abtest/base
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/leaf3
timeout 1500 python -m pytest tests -x -q -m gpu -p no:cacheprovider > gpurun_out/leaf3/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/leaf3/gpu_tests.log
tail -3 gpurun_out/leaf3/gpu_tests.log
for gspec in grid:256 road:4900 path:1e8 rmat:22 cat:20; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default,noleaf,default,noleaf >> gpurun_out/leaf3/ab.jsonl 2>> gpurun_out/leaf3/ab.err
  (cd abtest/base && timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "base"/' >> ../../gpurun_out/leaf3/ab.jsonl 2>> ../../gpurun_out/leaf3/ab.err)
done
timeout 900 python scripts/diag.py --graph rmat:22 --roots 1 --reps 1 --timeline 5 --variants default >> gpurun_out/leaf3/tl.jsonl 2>> gpurun_out/leaf3/ab.err
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/leaf3/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
for l in open('gpurun_out/leaf3/tl.jsonl'):
    r=json.loads(l); print(r['ms'], r['claims_by_5pct'])
PY
tail -3 gpurun_out/leaf3/ab.err
