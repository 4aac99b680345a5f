cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python scripts/diag.py --graph cat:262144 --roots 1 --reps 1 --variants w0,w0nospill > gpurun_out/diag19_cat.jsonl 2> gpurun_out/diag19.err
python - <<'PY'
import json
for f in ['gpurun_out/diag19_cat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(json.dumps({k: d[k] for k in ['variant','ms','claims','windows','flushes','spills','refills','intra','inter','cyc_total','cyc_per_window']}))
PY
tail -2 gpurun_out/diag19.err
