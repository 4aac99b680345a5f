cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --variants det32,det_nospec > gpurun_out/diag11_det.jsonl 2> gpurun_out/diag11.err
timeout 300 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --variants default > gpurun_out/diag11_road.jsonl 2>> gpurun_out/diag11.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 1 --reps 1 --variants default,det32 > gpurun_out/diag11_rmat.jsonl 2>> gpurun_out/diag11.err
python - <<'PY'
import json
for f in ['gpurun_out/diag11_det.jsonl','gpurun_out/diag11_road.jsonl','gpurun_out/diag11_rmat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'w/c',d['windows_per_claim'],'cyc/win',d['cyc_per_window'])
PY
tail -2 gpurun_out/diag11.err
