# A/B: hierarchical termination counters (working tree) vs abtest/base
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/term
timeout 1500 python -m pytest tests -x -q -m gpu -p no:cacheprovider > gpurun_out/term/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/term/gpu_tests.log
tail -3 gpurun_out/term/gpu_tests.log
for gspec in grid:256 road:4900 path:1e8 rmat:22 cat:20; do
  for rep in 1 2; do
    timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default | sed 's/"variant": "default"/"variant": "new"/' >> gpurun_out/term/ab.jsonl 2>> gpurun_out/term/ab.err
    (cd abtest/base && timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants specpop | sed 's/"variant": "specpop"/"variant": "base"/' >> ../../gpurun_out/term/ab.jsonl 2>> ../../gpurun_out/term/ab.err)
  done
done
timeout 900 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --variants default >> gpurun_out/term/stats.jsonl 2>> gpurun_out/term/ab.err
(cd abtest/base && timeout 900 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --variants specpop >> ../../gpurun_out/term/stats.jsonl 2>> ../../gpurun_out/term/ab.err)
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/term/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
for l in open('gpurun_out/term/stats.jsonl'):
    r=json.loads(l); print({k: r[k] for k in ('variant','ms','util','claims','intra','inter','attempts','scans','spills','flushes','refills')})
PY
tail -3 gpurun_out/term/ab.err
