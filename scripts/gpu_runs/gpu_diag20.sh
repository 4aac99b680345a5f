cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests20.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests20.log
tail -2 gpurun_out/gpu_tests20.log
timeout 900 python scripts/diag.py --graph road:4900 --roots 4 --reps 2 --nostats --variants default,bmin256,bmin1k,bmax512,bmax8k > gpurun_out/diag20_road.jsonl 2> gpurun_out/diag20.err
python - <<'PY'
import json, collections
agg = collections.defaultdict(list)
for l in open('gpurun_out/diag20_road.jsonl'):
    d=json.loads(l); agg[d['variant']].append(d['ms']); print(d['variant'], d['root'], d['ms'])
for k,v in agg.items(): print('MEAN', k, round(sum(v)/len(v),2))
PY
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench20.json 2> gpurun_out/bench20.err
python -c "import json; d=json.load(open('gpurun_out/bench20.json')); print(d['value'], d['ms_per_dfs'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'], 'upload', d['e2e']['with_upload']['value'], d['e2e']['with_upload']['ms_per_step'], 'cpu', d['cpu_baseline']['value'])"
