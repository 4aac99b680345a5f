cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests21.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests21.log
tail -2 gpurun_out/gpu_tests21.log
timeout 900 python scripts/diag.py --graph road:4900 --roots 4 --reps 2 --nostats --variants default > gpurun_out/diag21_road.jsonl 2> gpurun_out/diag21.err
timeout 900 python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --nostats --variants det32 >> gpurun_out/diag21_road.jsonl 2>> gpurun_out/diag21.err
python - <<'PY'
import json, collections
agg = collections.defaultdict(list)
for l in open('gpurun_out/diag21_road.jsonl'):
    d=json.loads(l); agg[d['graph']+d['variant']].append(d['ms']); print(d['graph'], d['variant'], d['root'], d['ms'])
for k,v in agg.items(): print('MEAN', k, round(sum(v)/len(v),2))
PY
