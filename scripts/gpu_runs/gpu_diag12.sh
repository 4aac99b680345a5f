cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests12.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests12.log
tail -3 gpurun_out/gpu_tests12.log
timeout 300 python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --variants det32,det_p1,det_p2,det_p1nospec > gpurun_out/diag12_det.jsonl 2> gpurun_out/diag12.err
timeout 600 python scripts/diag.py --graph road:4900 --roots 3 --reps 2 --variants default,p1,p2,p1nospec > gpurun_out/diag12_road.jsonl 2>> gpurun_out/diag12.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 2 --reps 2 --variants default,p1 > gpurun_out/diag12_rmat.jsonl 2>> gpurun_out/diag12.err
python - <<'PY'
import json
for f in ['gpurun_out/diag12_det.jsonl','gpurun_out/diag12_road.jsonl','gpurun_out/diag12_rmat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'fail',d['failed'],'cyc/win',d['cyc_per_window'])
PY
tail -2 gpurun_out/diag12.err
