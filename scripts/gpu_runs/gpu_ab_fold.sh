cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/fold
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider > gpurun_out/fold/parity.log 2>&1; echo "parity rc=$?" >> gpurun_out/fold/parity.log
tail -3 gpurun_out/fold/parity.log
for gspec in road:4900 rmat:22 path:1e8 grid:256; do
  for rep in 1 2; do
  timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants default,bmax512,bmax8k,bmin256 >> gpurun_out/fold/ab.jsonl 2>> gpurun_out/fold/ab.err
  (cd abtest/base && timeout 900 python scripts/diag.py --graph $gspec --roots 3 --reps 1 --nostats --variants early2st8 | sed 's/"variant": "early2st8"/"variant": "base"/' >> ../../gpurun_out/fold/ab.jsonl 2>> ../../gpurun_out/fold/ab.err)
  done
done
timeout 300 python scripts/diag.py --graph path:1e6 --roots 1 --reps 3 --nostats --variants det >> gpurun_out/fold/ab.jsonl 2>> gpurun_out/fold/ab.err
(cd abtest/base && timeout 300 python scripts/diag.py --graph path:1e6 --roots 1 --reps 3 --nostats --variants detearly | sed 's/"variant": "detearly"/"variant": "base"/' >> ../../gpurun_out/fold/ab.jsonl 2>> ../../gpurun_out/fold/ab.err)
python - <<'PY'
import json, collections
d=collections.defaultdict(list)
for l in open('gpurun_out/fold/ab.jsonl'):
    r=json.loads(l); d[(r['graph'],r['variant'])].append(r['ms'])
for k,v in sorted(d.items()): print(k, 'mean ms', round(sum(v)/len(v),3), v)
PY
tail -3 gpurun_out/fold/ab.err
