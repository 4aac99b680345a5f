cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests10.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests10.log
tail -4 gpurun_out/gpu_tests10.log
timeout 300 python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --variants det32,det_nospec > gpurun_out/diag10_det.jsonl 2> gpurun_out/diag10.err
timeout 600 python scripts/diag.py --graph cat:262144 --roots 1 --reps 1 --variants default,det32 > gpurun_out/diag10_cat.jsonl 2>> gpurun_out/diag10.err
timeout 900 python scripts/diag.py --graph road:4900 --roots 3 --reps 2 --timeline 20 --variants default,spec0 > gpurun_out/diag10_road.jsonl 2>> gpurun_out/diag10.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 2 --reps 2 --timeline 5 --variants default,A16 > gpurun_out/diag10_rmat.jsonl 2>> gpurun_out/diag10.err
python - <<'PY'
import json
for f in ['gpurun_out/diag10_det.jsonl','gpurun_out/diag10_cat.jsonl','gpurun_out/diag10_road.jsonl','gpurun_out/diag10_rmat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'busy',d.get('busy_mean'),d.get('busy_by_5pct'))
PY
tail -2 gpurun_out/diag10.err
