cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x -k "stress" > gpurun_out/eager_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/eager_tests.log; tail -2 gpurun_out/eager_tests.log
timeout 900 python scripts/diag.py --graph road:4900 --roots 4 --reps 2 --nostats --timeline 20 --variants default,eager > gpurun_out/diag_eager.jsonl 2> gpurun_out/diag_eager.err
timeout 900 python scripts/diag.py --graph path:1e7 --roots 2 --reps 2 --nostats --variants default,eager >> gpurun_out/diag_eager.jsonl 2>> gpurun_out/diag_eager.err
timeout 900 python scripts/diag.py --graph cat:262144 --roots 1 --reps 1 --nostats --variants default,eager >> gpurun_out/diag_eager.jsonl 2>> gpurun_out/diag_eager.err
timeout 900 python scripts/diag.py --graph grid:256 --roots 2 --reps 3 --nostats --variants default,eager >> gpurun_out/diag_eager.jsonl 2>> gpurun_out/diag_eager.err
python - <<'PY'
import json, collections
agg = collections.defaultdict(list)
for l in open('gpurun_out/diag_eager.jsonl'):
    d=json.loads(l); agg[d['graph']+' '+d['variant']].append(d['ms']); print(d['graph'], d['variant'], d['root'], d['ms'], d.get('busy_by_5pct'))
for k,v in agg.items(): print('MEAN', k, round(sum(v)/len(v),2))
PY
