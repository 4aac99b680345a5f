cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/tl2
timeout 600 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --timeline 200 --variants default > gpurun_out/tl2/road_tl.jsonl 2>> gpurun_out/tl2/err.log
timeout 600 python scripts/diag.py --graph rmat:22 --roots 2 --reps 1 --timeline 50 --variants default > gpurun_out/tl2/rmat_tl.jsonl 2>> gpurun_out/tl2/err.log
timeout 600 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --variants default,A16 >> gpurun_out/tl2/road_stats.jsonl 2>> gpurun_out/tl2/err.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 2 -c 1 -o gpurun_out/tl2/prof_road24m python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/tl2/ncu_full.log 2>&1
python - <<'PY'
import json
for f in ('road_tl','rmat_tl','road_stats'):
    for l in open(f'gpurun_out/tl2/{f}.jsonl'):
        r=json.loads(l); print(f, r['variant'], r['ms'], 'util', r['util'], 'busy_mean', r.get('busy_mean'), r.get('busy_by_5pct'), r.get('claims_by_5pct'))
PY
tail -3 gpurun_out/tl2/err.log
