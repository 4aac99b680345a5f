# group steals: parity tests, sweeps, ncu of the walker kernel on road24m
timeout 1200 python -m pytest tests/test_gpu_walker.py -q -x --timeout 120 -rf > gpurun_out/pytest_walker4.log 2>&1; echo walker tests rc=$?
tail -5 gpurun_out/pytest_walker4.log
L=paper_conf_ppopp_niul0c26_b200/libdfs.so
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --reps 3 --steps 6 \
  --variant "" --variant "walker_lanes=8,records=0,steal_period=16" --variant "walker_lanes=8,records=0,steal_period=1" \
  --variant "walker_lanes=16,records=0,steal_period=16" --variant "walker_lanes=4,steal_period=16" > gpurun_out/ab_g_road.jsonl 2>&1
grep lib gpurun_out/ab_g_road.jsonl || tail -20 gpurun_out/ab_g_road.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --config road24m --reps 2 --batch 64 \
  --variant "" --variant "walker_lanes=8,records=0,steal_period=16" --variant "walker_lanes=8,records=0,steal_period=1" \
  --variant "walker_lanes=16,records=0,steal_period=16" --variant "walker_lanes=4,steal_period=16" > gpurun_out/ab_g_batch.jsonl 2>&1
grep lib gpurun_out/ab_g_batch.jsonl || tail -20 gpurun_out/ab_g_batch.jsonl
timeout 600 python scripts/ab_libs.py --libs $L --config path100m --reps 3 --steps 4 \
  --variant "" --variant "walker_lanes=8,records=0,steal_period=16" --variant "walker_lanes=4,steal_period=16" > gpurun_out/ab_g_path.jsonl 2>&1
grep lib gpurun_out/ab_g_path.jsonl || tail -20 gpurun_out/ab_g_path.jsonl
timeout 900 ncu --set full --import-source on --clock-control none -k regex:dfs_walker_kernel --launch-skip 1 -c 1 \
  -o gpurun_out/ncu_walker_road python scripts/ncu_run.py --config road24m --set walker_lanes=8 --set records=0 --set steal_period=16 > gpurun_out/ncu_walker_road.log 2>&1; echo ncu rc=$?
tail -3 gpurun_out/ncu_walker_road.log
