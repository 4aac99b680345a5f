cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests5.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests5.log
tail -4 gpurun_out/gpu_tests5.log
timeout 300 python scripts/diag.py --graph grid:256 --roots 1 --reps 1 --variants det32,det128,h2c2w32,h2c2w128 > gpurun_out/diag5_grid.jsonl 2> gpurun_out/diag5.err
timeout 300 python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --variants det32,det128 > gpurun_out/diag5_roaddet.jsonl 2>> gpurun_out/diag5.err
timeout 900 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --timeline 20 --variants h2c2w32,h2c2w128,h4c4w32,h4c4w128 > gpurun_out/diag5_road.jsonl 2>> gpurun_out/diag5.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 1 --reps 1 --timeline 5 --variants h2c2w32,h2c2w128,h4c4w128 > gpurun_out/diag5_rmat.jsonl 2>> gpurun_out/diag5.err
python - <<'PY'
import json
for f in ['gpurun_out/diag5_grid.jsonl','gpurun_out/diag5_roaddet.jsonl','gpurun_out/diag5_road.jsonl','gpurun_out/diag5_rmat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'w/c',d['windows_per_claim'],'sp',d['spills'],'inter',d['inter'],'intra',d['intra'],'busy',d.get('busy_mean'),d.get('busy_by_5pct'))
PY
tail -3 gpurun_out/diag5.err
