cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/l2p
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider -k "stress or deterministic or bulk" > gpurun_out/l2p/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/l2p/parity.log
tail -3 gpurun_out/l2p/parity.log
for g in rmat:24 road:4900 path:1e8; do
for rep in 1 2; do
  (cd abtest/base && timeout 600 python scripts/diag.py --graph $g --roots 3 --reps 1 --nostats --variants default | sed "s/\"variant\": \"default\"/\"variant\": \"base\"/" >> ../../gpurun_out/l2p/diag.jsonl 2>> ../../gpurun_out/l2p/err.log)
  timeout 600 python scripts/diag.py --graph $g --roots 3 --reps 1 --nostats --variants default,l2p32,l2p64,l2p96 >> gpurun_out/l2p/diag.jsonl 2>> gpurun_out/l2p/err.log
done
done
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/l2p/diag.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
python -c "import torch; p=torch.cuda.get_device_properties(0); print('persisting max', p.persisting_l2_cache_max_size if hasattr(p,'persisting_l2_cache_max_size') else '?', 'L2', p.L2_cache_size)"
tail -2 gpurun_out/l2p/err.log
