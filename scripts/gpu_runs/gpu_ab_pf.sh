# A/B: 128-wide step, row_ptr pairs prefetched with the probes for the first 8 (default) / 16 / 32 positions
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/pf
for v in pf4 pf8; do (cd abtest/$v && timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "stress or parallel or bit_exact" > ../../gpurun_out/pf/parity_$v.log 2>&1; tail -1 ../../gpurun_out/pf/parity_$v.log); done
for rep in 1 2; do
  for v in head pf4 pf8; do
    (cd abtest/$v && timeout 600 python bench.py --config rmat24 --steps 8 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > ../../gpurun_out/pf/${v}_rmat24_$rep.json 2>/dev/null)
  done
done
for v in head pf4 pf8; do
  (cd abtest/$v && timeout 600 python scripts/diag.py --graph rmat:22 --roots 3 --reps 1 --nostats --variants default,default > ../../gpurun_out/pf/${v}_rmat22.jsonl 2>> ../../gpurun_out/pf/err.log)
done
for f in gpurun_out/pf/*.json; do python -c "import json,sys; d=json.load(open('$f')); print('$f', d['value'], d['ms_per_dfs'], d['ms_per_dfs_median'])"; done
for f in gpurun_out/pf/*_rmat22.jsonl; do python -c "
import json; v=[json.loads(l)['ms'] for l in open('$f')]; print('$f', round(sum(v)/len(v),3), v)"; done
