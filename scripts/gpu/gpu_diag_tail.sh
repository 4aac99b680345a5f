# RMAT serial tail: windows vs claims over time (STATS build timeline), then the GPU test suite
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/tail
timeout 600 python scripts/diag.py --graph rmat:24 --roots 2 --reps 1 --timeline 100 --variants default > gpurun_out/tail/diag_rmat24.jsonl 2> gpurun_out/tail/err.log
timeout 600 python scripts/diag.py --graph rmat:22 --roots 1 --reps 1 --timeline 25 --variants default > gpurun_out/tail/diag_rmat22.jsonl 2>> gpurun_out/tail/err.log
timeout 600 python scripts/diag.py --graph road:4900 --roots 1 --reps 1 --timeline 100 --variants default > gpurun_out/tail/diag_road.jsonl 2>> gpurun_out/tail/err.log
python - <<'PY'
import json, glob
for f in sorted(glob.glob('gpurun_out/tail/diag_*.jsonl')):
    for l in open(f):
        d=json.loads(l); print(d['graph'], d['root'], d['ms'], d['n_visited'], 'windows', d.get('windows'))
        for k in ('busy_by_5pct','claims_by_5pct','windows_by_5pct'): print(' ', k, d.get(k))
PY
tail -3 gpurun_out/tail/err.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/tail/gpu_tests.log 2>&1; tail -3 gpurun_out/tail/gpu_tests.log
