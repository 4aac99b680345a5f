cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests2.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests2.log
tail -3 gpurun_out/gpu_tests2.log
timeout 900 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --variants default,paper,nospill,leader,h8c8,h16c16,h16c32,h8c32,h4c8,h8c8i128,h8c8i8,h8c8w16,hot8,h8c16 > gpurun_out/diag2_road.jsonl 2> gpurun_out/diag2_road.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 2 --reps 1 --variants default,paper,h8c8,h16c16,h16c32 > gpurun_out/diag2_rmat.jsonl 2>> gpurun_out/diag2_road.err
python - <<'PY'
import json
for f in ['gpurun_out/diag2_road.jsonl','gpurun_out/diag2_rmat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],d['util'],d['us_per_claim_per_warp'],'spills',d['spills'],'inter',d['inter'],'intra',d['intra'])
PY
tail -3 gpurun_out/diag2_road.err
