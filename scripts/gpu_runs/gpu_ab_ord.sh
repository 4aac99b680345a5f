# A/B: 128-wide step issues its probes before the speculative claim (no spill store waiting on the atomic)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ord
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/ord/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/ord/parity.log
tail -3 gpurun_out/ord/parity.log
for rep in 1 2 3; do
  timeout 600 python bench.py --config rmat24 --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/ord/head_rmat24_$rep.json 2>/dev/null
  (cd abtest/base && timeout 600 python bench.py --config rmat24 --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > ../../gpurun_out/ord/base_rmat24_$rep.json 2>/dev/null)
done
timeout 600 python scripts/diag.py --graph rmat:22 --roots 3 --reps 1 --nostats --variants default,spec128,default,spec128,default,spec128 > gpurun_out/ord/head_rmat22.jsonl 2>> gpurun_out/ord/err.log
(cd abtest/base && timeout 600 python scripts/diag.py --graph rmat:22 --roots 3 --reps 1 --nostats --variants default,default,default > ../../gpurun_out/ord/base_rmat22.jsonl 2>> ../../gpurun_out/ord/err.log)
for f in gpurun_out/ord/*.json; do python -c "import json,sys; d=json.load(open('$f')); print('$f', d['value'], d['ms_per_dfs'], d['ms_per_dfs_median'])"; done
timeout 600 python scripts/diag.py --graph rmat:24 --roots 3 --reps 1 --nostats --variants default,spec128,default,spec128 > gpurun_out/ord/head_rmat24_spec.jsonl 2>> gpurun_out/ord/err.log
for f in gpurun_out/ord/*.jsonl; do python -c "
import json; import collections; d=collections.defaultdict(list)
for l in open('$f'): r=json.loads(l); d[r['variant']].append(r['ms'])
for k,v in d.items(): print('$f', k, round(sum(v)/len(v),3), v)"; done
tail -3 gpurun_out/ord/err.log
