cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/cat2
timeout 600 python scripts/diag.py --graph cat:20 --roots 1 --reps 1 --variants w0,w0nospill,w0nointra >> gpurun_out/cat2/diag.jsonl 2>> gpurun_out/cat2/err.log
timeout 600 python scripts/diag.py --graph path:1e6 --roots 1 --reps 1 --variants w0det >> gpurun_out/cat2/diag.jsonl 2>> gpurun_out/cat2/err.log
timeout 600 python scripts/diag.py --graph cat:16 --roots 1 --reps 1 --variants w0det >> gpurun_out/cat2/diag.jsonl 2>> gpurun_out/cat2/err.log
timeout 600 python scripts/diag.py --graph cat:20 --roots 1 --reps 1 --nostats --variants default,nospill,pb4,pb16,nointra >> gpurun_out/cat2/diag.jsonl 2>> gpurun_out/cat2/err.log
python - <<'PY'
import json
for l in open('gpurun_out/cat2/diag.jsonl'):
    r=json.loads(l); print(r['graph'], r['variant'], r['ms'], 'win', r['windows'], 'claims', r['claims'], 'fl', r['flushes'], 'sp', r['spills'], 'cyc/win', r['cyc_per_window'], 'intra', r['intra'], 'failed', r['failed'])
PY
tail -3 gpurun_out/cat2/err.log
