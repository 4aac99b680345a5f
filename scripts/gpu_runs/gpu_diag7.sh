cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests7.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests7.log
tail -4 gpurun_out/gpu_tests7.log
timeout 300 python scripts/diag.py --graph road:1024 --roots 1 --reps 1 --variants det16 > gpurun_out/diag7_roaddet.jsonl 2> gpurun_out/diag7.err
timeout 900 python scripts/diag.py --graph road:4900 --roots 2 --reps 1 --timeline 20 --variants A,A16,A24,A8,B16,A16nospec,A16b8k > gpurun_out/diag7_road.jsonl 2>> gpurun_out/diag7.err
timeout 300 python scripts/diag.py --graph rmat:22 --roots 1 --reps 1 --timeline 5 --variants A,A16,B16,A16nospec > gpurun_out/diag7_rmat.jsonl 2>> gpurun_out/diag7.err
python - <<'PY'
import json
for f in ['gpurun_out/diag7_roaddet.jsonl','gpurun_out/diag7_road.jsonl','gpurun_out/diag7_rmat.jsonl']:
    for l in open(f):
        d=json.loads(l); print(d['graph'],d['variant'],d['root'],d['ms'],d['gteps'],'util',d['util'],'us/claim',d['us_per_claim_per_warp'],'w/c',d['windows_per_claim'],'fail',d['failed'],'sp',d['spills'],'inter',d['inter'],'intra',d['intra'],'busy',d.get('busy_mean'),d.get('busy_by_5pct'))
PY
tail -3 gpurun_out/diag7.err
