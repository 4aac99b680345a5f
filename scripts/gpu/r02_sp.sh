# walker kernel steal_period sweep (batch + path)
set -x
L=paper_conf_ppopp_niul0c26_b200/libdfs.so
timeout 900 python scripts/ab_libs.py --libs $L --variant "" --variant steal_period=32 --variant steal_period=64 --variant steal_period=128 --config road24m --batch 64 --reps 5 > gpurun_out/ab_sp_batch.jsonl 2>&1
grep -h lib gpurun_out/ab_sp_batch.jsonl || tail -5 gpurun_out/ab_sp_batch.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --variant "" --variant steal_period=32 --variant steal_period=64 --config path100m --reps 3 --steps 2 > gpurun_out/ab_sp_path.jsonl 2>&1
grep -h lib gpurun_out/ab_sp_path.jsonl || tail -5 gpurun_out/ab_sp_path.jsonl
timeout 900 python bench.py --config grid256 --steps 3 --warmup 3 --cpu-seconds 1 > gpurun_out/bench_grid_span.json 2>gpurun_out/bench_grid_span.err; echo bench rc=$?
python -c "import json; d=json.loads(open('gpurun_out/bench_grid_span.json').read().strip().splitlines()[-1]); print(d['span'])"
