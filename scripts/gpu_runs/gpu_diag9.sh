cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests9.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests9.log
tail -4 gpurun_out/gpu_tests9.log
timeout 900 python scripts/diag.py --graph road:4900 --roots 3 --reps 2 --timeline 20 --variants default,nohalf,h1c1,h1c2,h4c4,h1c1nohalf > gpurun_out/diag9_road.jsonl 2> gpurun_out/diag9.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 2 --reps 2 --timeline 5 --variants default,nohalf,h1c1,h1c1nohalf > gpurun_out/diag9_rmat.jsonl 2>> gpurun_out/diag9.err
python - <<'PY'
import json
for f in ['gpurun_out/diag9_road.jsonl','gpurun_out/diag9_rmat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'intra',d['intra'],'inter',d['inter'],'busy',d.get('busy_mean'),d.get('busy_by_5pct'))
PY
