# A/B: scan assist (dfs_options.scan_assist) and the rebuilt default kernel vs HEAD (abtest/base)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/assist
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/assist/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/assist/parity.log
tail -3 gpurun_out/assist/parity.log
for rep in 1 2; do
for c in rmat24 road24m; do
  timeout 600 python bench.py --config $c --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/assist/head_${c}_$rep.json 2>/dev/null
  (cd abtest/base && timeout 600 python bench.py --config $c --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > ../../gpurun_out/assist/base_${c}_$rep.json 2>/dev/null)
done
done
timeout 600 python scripts/diag.py --graph rmat:24 --roots 3 --reps 1 --nostats --variants default,assist1,assist4,default,assist1,assist4 >> gpurun_out/assist/diag.jsonl 2>> gpurun_out/assist/err.log
timeout 600 python scripts/diag.py --graph rmat:22 --roots 3 --reps 1 --nostats --variants default,assist4,default,assist4 >> gpurun_out/assist/diag.jsonl 2>> gpurun_out/assist/err.log
for f in gpurun_out/assist/*.json; do python -c "import json,sys; d=json.load(open('$f')); print('$f', d['value'], d['ms_per_dfs'], d['ms_per_dfs_median'])"; done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/assist/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -3 gpurun_out/assist/err.log
