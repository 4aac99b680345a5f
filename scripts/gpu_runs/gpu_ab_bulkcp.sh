cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/bulkcp
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/bulkcp/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "bulk or stress or deterministic" > gpurun_out/bulkcp/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/bulkcp/parity.log
tail -3 gpurun_out/bulkcp/parity.log
for gspec in road:4900 rmat:22 path:1e8 cat:20; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 2 --reps 1 --nostats --variants default,bulk_copy,v1,bulk_copy_v1,sp8,sp16,sp64,default,bulk_copy,sp8,sp16 >> gpurun_out/bulkcp/ab.jsonl 2>> gpurun_out/bulkcp/ab.err
done
timeout 300 python scripts/diag.py --graph grid:256 --roots 1 --reps 3 --nostats --variants det,detbulk,det,detbulk >> gpurun_out/bulkcp/ab.jsonl 2>> gpurun_out/bulkcp/ab.err
timeout 600 python scripts/diag.py --graph road:4900 --roots 1 --reps 1 --variants default,bulk_copy >> gpurun_out/bulkcp/stats.jsonl 2>> gpurun_out/bulkcp/ab.err
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/bulkcp/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
for l in open('gpurun_out/bulkcp/stats.jsonl'):
    r=json.loads(l); print(r['variant'], r['ms'], 'flushes', r['flushes'], 'refills', r['refills'], 'spills', r['spills'])
PY
tail -3 gpurun_out/bulkcp/ab.err
