# vertex records in the walker kernel: parity tests, then A/B on road (single + batch) and path
timeout 1200 python -m pytest tests/test_gpu_walker.py -q -x --timeout 120 -rf > gpurun_out/pytest_walker3.log 2>&1; echo walker tests rc=$?
tail -5 gpurun_out/pytest_walker3.log
L=paper_conf_ppopp_niul0c26_b200/libdfs.so
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --reps 3 --steps 6 \
  --variant "" --variant "walker_lanes=8,records=0,steal_period=1024" --variant "walker_lanes=8,steal_period=1024" \
  --variant "walker_lanes=16,records=0,steal_period=16" --variant "walker_lanes=16,steal_period=16" \
  --variant "walker_lanes=16,steal_period=1024" > gpurun_out/ab_rec_road.jsonl 2>&1
grep lib gpurun_out/ab_rec_road.jsonl || tail -20 gpurun_out/ab_rec_road.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --reps 2 --batch 64 \
  --variant "" --variant "walker_lanes=8,records=0" --variant "walker_lanes=8" --variant "walker_lanes=16" \
  --variant "walker_lanes=8,concurrency=4" --variant "walker_lanes=8,steal_period=16" --variant "walker_lanes=4" > gpurun_out/ab_rec_batch.jsonl 2>&1
grep lib gpurun_out/ab_rec_batch.jsonl || tail -20 gpurun_out/ab_rec_batch.jsonl
timeout 600 python scripts/ab_libs.py --libs $L --config path100m --reps 3 --steps 4 \
  --variant "" --variant "walker_lanes=8" --variant "walker_lanes=8,records=0" --variant "walker_lanes=4" > gpurun_out/ab_rec_path.jsonl 2>&1
grep lib gpurun_out/ab_rec_path.jsonl || tail -20 gpurun_out/ab_rec_path.jsonl
