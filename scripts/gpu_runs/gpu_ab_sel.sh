# A/B: leaf check of the 128-wide step with selects instead of a dynamically indexed local array
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/sel
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/sel/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/sel/parity.log
tail -3 gpurun_out/sel/parity.log
for rep in 1 2 3; do
  timeout 600 python bench.py --config rmat24 --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/sel/head_rmat24_$rep.json 2>/dev/null
  (cd abtest/base && timeout 600 python bench.py --config rmat24 --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > ../../gpurun_out/sel/base_rmat24_$rep.json 2>/dev/null)
done
timeout 600 python scripts/diag.py --graph rmat:22 --roots 3 --reps 1 --nostats --variants default,default,default > gpurun_out/sel/head_rmat22.jsonl 2>> gpurun_out/sel/err.log
(cd abtest/base && timeout 600 python scripts/diag.py --graph rmat:22 --roots 3 --reps 1 --nostats --variants default,default,default > ../../gpurun_out/sel/base_rmat22.jsonl 2>> ../../gpurun_out/sel/err.log)
for f in gpurun_out/sel/*.json; do python -c "import json,sys; d=json.load(open('$f')); print('$f', d['value'], d['ms_per_dfs'], d['ms_per_dfs_median'])"; done
for f in gpurun_out/sel/*_rmat22.jsonl; do python -c "
import json; v=[json.loads(l)['ms'] for l in open('$f')]; print('$f', round(sum(v)/len(v),3), v)"; done
tail -3 gpurun_out/sel/err.log
