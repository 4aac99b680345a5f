# 2-lane walkers: parity tests (walker + stack script), then A/B on batch / path / road
timeout 1500 python -m pytest tests/test_gpu_walker.py tests/test_gpu_stack_script.py -q -x --timeout 150 -rf > gpurun_out/pytest_g2.log 2>&1; echo walker tests rc=$?
tail -5 gpurun_out/pytest_g2.log
L=paper_conf_ppopp_niul0c26_b200/libdfs.so
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --reps 2 --batch 64 \
  --variant "" --variant "walker_lanes=2" --variant "walker_lanes=2,concurrency=12" --variant "walker_lanes=2,steal_period=64" > gpurun_out/ab_g2_batch.jsonl 2>&1
grep lib gpurun_out/ab_g2_batch.jsonl || tail -20 gpurun_out/ab_g2_batch.jsonl
timeout 600 python scripts/ab_libs.py --libs $L --config path100m --reps 3 --steps 4 \
  --variant "" --variant "walker_lanes=2" > gpurun_out/ab_g2_path.jsonl 2>&1
grep lib gpurun_out/ab_g2_path.jsonl || tail -20 gpurun_out/ab_g2_path.jsonl
