# walker kernel: parity tests, then A/B of the warp kernel vs walkers on road24m / path / grid
timeout 900 python -m pytest tests/test_gpu_walker.py -q -x --timeout 120 -rf > gpurun_out/pytest_walker.log 2>&1; echo walker tests rc=$?
tail -15 gpurun_out/pytest_walker.log
L=paper_conf_ppopp_niul0c26_b200/libdfs.so
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --reps 3 --steps 6 \
  --variant "" --variant "walker_lanes=16" --variant "walker_lanes=8" --variant "walker_lanes=4" \
  --variant "walker_lanes=8,steal_period=4" --variant "walker_lanes=4,steal_period=4" > gpurun_out/ab_walker_road.jsonl 2>&1
grep lib gpurun_out/ab_walker_road.jsonl || tail -20 gpurun_out/ab_walker_road.jsonl
timeout 600 python scripts/ab_libs.py --libs $L --config road24m --reps 2 --batch 64 \
  --variant "" --variant "walker_lanes=8" --variant "walker_lanes=4" --variant "walker_lanes=8,concurrency=16" --variant "walker_lanes=4,concurrency=16" --variant "concurrency=16" > gpurun_out/ab_walker_batch.jsonl 2>&1
grep lib gpurun_out/ab_walker_batch.jsonl || tail -20 gpurun_out/ab_walker_batch.jsonl
for c in path100m grid256 caterpillar; do
timeout 600 python scripts/ab_libs.py --libs $L --config $c --reps 3 --steps 4 \
  --variant "" --variant "walker_lanes=8" --variant "walker_lanes=4" > gpurun_out/ab_walker_$c.jsonl 2>&1
grep lib gpurun_out/ab_walker_$c.jsonl || tail -20 gpurun_out/ab_walker_$c.jsonl
done
