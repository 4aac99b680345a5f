cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests4.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests4.log
tail -2 gpurun_out/gpu_tests4.log
timeout 900 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --timeline 20 --variants h4c4,h2c2,h2c4,h4c2,h2c2w16,h2c2i1,h6c2 > gpurun_out/diag4_road.jsonl 2> gpurun_out/diag4_road.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 2 --reps 1 --timeline 5 --variants default,h4c4,h2c2 > gpurun_out/diag4_rmat.jsonl 2>> gpurun_out/diag4_road.err
timeout 300 python scripts/diag.py --graph grid:256 --roots 1 --reps 1 --variants det,h4c4,h2c2 > gpurun_out/diag4_grid.jsonl 2>> gpurun_out/diag4_road.err
python - <<'PY'
import json
for f in ['gpurun_out/diag4_road.jsonl','gpurun_out/diag4_rmat.jsonl','gpurun_out/diag4_grid.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'w/c',d['windows_per_claim'],'sp',d['spills'],'inter',d['inter'],'intra',d['intra'],'busy',d.get('busy_mean'),d.get('busy_by_5pct'))
PY
tail -3 gpurun_out/diag4_road.err
