cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/cl
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/cl/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/cl/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/cl/parity.log
tail -3 gpurun_out/cl/parity.log
for gspec in road:4900 rmat:22 grid:256 path:1e8 cat:20; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default,cl2,cl4,cl8,default,cl2,cl4 >> gpurun_out/cl/ab.jsonl 2>> gpurun_out/cl/ab.err
done
timeout 600 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --variants default,cl2stats >> gpurun_out/cl/stats.jsonl 2>> gpurun_out/cl/ab.err
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/cl/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
for l in open('gpurun_out/cl/stats.jsonl'):
    r=json.loads(l); print(r['variant'], r['ms'], 'util', r['util'], 'intra', r['intra'], 'inter', r['inter'], 'cl', r.get('cl'), 'blocks', r.get('blocks'))
PY
tail -3 gpurun_out/cl/ab.err
