cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python scripts/diag.py --graph rmat:22 --roots 1 --reps 1 --nostats --timeline 5 --variants default > gpurun_out/diag24.jsonl 2> gpurun_out/diag24.err
timeout 900 python scripts/diag.py --graph road:4900 --roots 1 --reps 1 --nostats --timeline 20 --variants default >> gpurun_out/diag24.jsonl 2>> gpurun_out/diag24.err
python - <<'PY'
import json
for l in open('gpurun_out/diag24.jsonl'):
    d=json.loads(l); print(d['graph'], d['ms'], d['n_visited']); print(' busy', d.get('busy_by_5pct')); print(' claims', d.get('claims_by_5pct'))
PY
tail -3 gpurun_out/diag24.err
