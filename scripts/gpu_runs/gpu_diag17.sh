cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python scripts/diag.py --graph road:4900 --roots 3 --reps 2 --variants default,pf,pfp1 > gpurun_out/diag17_road.jsonl 2> gpurun_out/diag17.err
timeout 600 python scripts/diag.py --graph cat:262144 --roots 1 --reps 1 --timeline 50 --variants default,nospill,pf,h4c4,pb8,b37 > gpurun_out/diag17_cat.jsonl 2>> gpurun_out/diag17.err
timeout 300 python scripts/diag.py --graph grid:256 --roots 2 --reps 3 --variants default,b37,b16,pf > gpurun_out/diag17_grid.jsonl 2>> gpurun_out/diag17.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 2 --reps 2 --variants default,pf > gpurun_out/diag17_rmat.jsonl 2>> gpurun_out/diag17.err
python - <<'PY'
import json
for f in ['gpurun_out/diag17_road.jsonl','gpurun_out/diag17_cat.jsonl','gpurun_out/diag17_grid.jsonl','gpurun_out/diag17_rmat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'spills',d['spills'],'intra',d['intra'],'cyc',d['cyc_per_window'],'busy',d.get('busy_mean'))
PY
tail -2 gpurun_out/diag17.err
