cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests6.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests6.log
tail -4 gpurun_out/gpu_tests6.log
timeout 300 python scripts/diag.py --graph grid:256 --roots 1 --reps 1 --variants det32,det_nospec,det_pb1,det_pb1_nospec > gpurun_out/diag6_grid.jsonl 2> gpurun_out/diag6.err
timeout 300 python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --variants det32,det_nospec,det_pb1,det_pb1_nospec > gpurun_out/diag6_roaddet.jsonl 2>> gpurun_out/diag6.err
timeout 900 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --timeline 20 --variants h2c2pb1,h2c2pb2,h2c2pb4,h2c2pb16,h2c2nospec,h4c4pb4 > gpurun_out/diag6_road.jsonl 2>> gpurun_out/diag6.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 1 --reps 1 --timeline 5 --variants h2c2pb4,h2c2nospec,h4c4pb4 > gpurun_out/diag6_rmat.jsonl 2>> gpurun_out/diag6.err
python - <<'PY'
import json
for f in ['gpurun_out/diag6_grid.jsonl','gpurun_out/diag6_roaddet.jsonl','gpurun_out/diag6_road.jsonl','gpurun_out/diag6_rmat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'w/c',d['windows_per_claim'],'fail',d['failed'],'sp',d['spills'],'inter',d['inter'],'intra',d['intra'],'busy',d.get('busy_mean'),d.get('busy_by_5pct'))
PY
tail -3 gpurun_out/diag6.err
