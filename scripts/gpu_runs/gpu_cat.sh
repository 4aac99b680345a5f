cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/cat
timeout 1200 python scripts/diag.py --graph cat:20 --roots 1 --reps 1 --nostats --variants default,pb4,pb16,nospill,spill128,spill1k,h4c4,bmin256,w0 > gpurun_out/cat/ab.jsonl 2> gpurun_out/cat/err
timeout 600 python scripts/diag.py --graph cat:16 --roots 1 --reps 1 --nostats --variants det,default >> gpurun_out/cat/ab.jsonl 2>> gpurun_out/cat/err
python - <<'PY'
import json
for l in open('gpurun_out/cat/ab.jsonl'):
    r=json.loads(l); print(r['graph'], r['variant'], r['ms'], {k: r[k] for k in ('claims','windows','flushes','refills','intra','inter','spills','attempts')})
PY
tail -2 gpurun_out/cat/err
