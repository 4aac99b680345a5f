cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests13.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests13.log
tail -3 gpurun_out/gpu_tests13.log
timeout 300 python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --variants det32,det_nospec,det_p1 > gpurun_out/diag13_det.jsonl 2> gpurun_out/diag13.err
timeout 600 python scripts/diag.py --graph road:4900 --roots 3 --reps 2 --variants default,p1,spec0 > gpurun_out/diag13_road.jsonl 2>> gpurun_out/diag13.err
python - <<'PY'
import json
for f in ['gpurun_out/diag13_det.jsonl','gpurun_out/diag13_road.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'fail',d['failed'],'cyc/win',d['cyc_per_window'])
PY
tail -2 gpurun_out/diag13.err
