cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/st
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/st/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "stress or deterministic" > gpurun_out/st/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/st/parity.log
tail -3 gpurun_out/st/parity.log
for gspec in road:4900 rmat:22 path:1e8 grid:256; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default,noearly,st2,st4,st8,default,noearly,st2,st4,st8 >> gpurun_out/st/ab.jsonl 2>> gpurun_out/st/ab.err
done
timeout 600 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --variants default,st4 >> gpurun_out/st/stats.jsonl 2>> gpurun_out/st/ab.err
timeout 600 python scripts/diag.py --graph cat:20 --roots 2 --reps 1 --nostats --variants default,noearly,st4 >> gpurun_out/st/ab.jsonl 2>> gpurun_out/st/ab.err
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/st/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
for l in open('gpurun_out/st/stats.jsonl'):
    r=json.loads(l); print(r['variant'], r['ms'], 'util', r['util'], 'intra', r['intra'], 'inter', r['inter'], 'attempts', r['attempts'], 'scans', r['scans'])
PY
tail -3 gpurun_out/st/ab.err
