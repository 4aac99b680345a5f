cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/dp
for g in road:4900 path:1e8 grid:256; do
  timeout 600 python scripts/diag.py --graph $g --roots 2 --reps 1 --variants default >> gpurun_out/dp/diag.jsonl 2>> gpurun_out/dp/err.log
done
python - <<'PY'
import json
for l in open('gpurun_out/dp/diag.jsonl'):
    r=json.loads(l); print(r['graph'], r['ms'], 'claims', r['claims'], 'windows', r['windows'], 'pops', r['pops'], 'dead', r['dead_pops'], 'failed', r['failed'], 'util', r['util'])
PY
tail -2 gpurun_out/dp/err.log
