# A/B: short-list speculation for 128-wide windows (speculate bit 4) on RMAT
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/specshort
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider  > gpurun_out/specshort/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/specshort/parity.log
tail -3 gpurun_out/specshort/parity.log
for c in rmat24 road24m; do
  timeout 600 python bench.py --config $c --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/specshort/head_${c}.json 2>/dev/null
  (cd abtest/base && timeout 600 python bench.py --config $c --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > ../../gpurun_out/specshort/base_${c}.json 2>/dev/null)
done
for f in gpurun_out/specshort/*.json; do python -c "import json,sys; d=json.load(open('$f')); print('$f', d['value'], d['ms_per_dfs'], d['ms_per_dfs_median'])"; done
timeout 900 python scripts/diag.py --graph rmat:24 --roots 3 --reps 1 --nostats --variants default,specshort,spec128,default,specshort,spec128 >> gpurun_out/specshort/diag.jsonl 2>> gpurun_out/specshort/err.log
timeout 600 python scripts/diag.py --graph rmat:22 --roots 3 --reps 1 --nostats --variants default,specshort,spec128,default,specshort,spec128 >> gpurun_out/specshort/diag.jsonl 2>> gpurun_out/specshort/err.log
timeout 600 python scripts/diag.py --graph rmat:24 --roots 1 --reps 1 --timeline 100 --variants specshort >> gpurun_out/specshort/timeline.jsonl 2>> gpurun_out/specshort/err.log
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/specshort/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
for l in open('gpurun_out/specshort/timeline.jsonl'):
    r=json.loads(l); print(r['ms'], r.get('busy_by_5pct')); print(r.get('claims_by_5pct'))
PY
tail -3 gpurun_out/specshort/err.log
