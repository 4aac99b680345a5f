cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/tl
timeout 900 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --nostats --timeline 20 --variants default > gpurun_out/tl/road.jsonl 2> gpurun_out/tl/err
timeout 900 python scripts/diag.py --graph cat:20 --roots 1 --reps 1 --timeline 50 --variants default > gpurun_out/tl/cat.jsonl 2>> gpurun_out/tl/err
timeout 900 python scripts/diag.py --graph rmat:22 --roots 2 --reps 1 --timeline 5 --variants default > gpurun_out/tl/rmat.jsonl 2>> gpurun_out/tl/err
python - <<'PY'
import json
for f in ('road','cat','rmat'):
    for l in open(f'gpurun_out/tl/{f}.jsonl'):
        d=json.loads(l); print(d['graph'], d['root'], d['ms'], 'util', d.get('util'), 'claims', d['claims'], 'intra', d['intra'], 'inter', d['inter'], 'spills', d['spills'])
        print('  busy blocks', d.get('busy_by_5pct')); print('  claims     ', d.get('claims_by_5pct'))
PY
