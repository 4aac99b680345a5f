cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/conc16
for rep in 1 2; do
for k in 8 12 16; do
  timeout 900 python bench.py --config batch1024 --warmup 3 --concurrency $k > gpurun_out/conc16/batch_k${k}_$rep.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/conc16/batch_k${k}_$rep.json')); print('batch k=$k rep $rep', d['value'], d['dfs_per_s'])"
done
done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -p no:cacheprovider -k concurrent > gpurun_out/conc16/parity.log 2>&1; tail -1 gpurun_out/conc16/parity.log
