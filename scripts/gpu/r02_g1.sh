# thread walkers (walker_lanes = 1) vs the 4-lane default: parity, batch, path, road single
set -x
timeout 600 python -m pytest tests/test_gpu_walker.py -q -x --timeout 120 -k "-1]" > gpurun_out/pytest_g1.log 2>&1; echo pytest rc=$?
tail -5 gpurun_out/pytest_g1.log
L=paper_conf_ppopp_niul0c26_b200/libdfs.so
timeout 600 python scripts/ab_libs.py --libs $L --variant walker_lanes=4 --variant walker_lanes=1 --config road24m --batch 64 --reps 3 > gpurun_out/ab_g1_batch.jsonl 2>&1
grep -h lib gpurun_out/ab_g1_batch.jsonl || tail -5 gpurun_out/ab_g1_batch.jsonl
timeout 600 python scripts/ab_libs.py --libs $L --variant walker_lanes=4 --variant walker_lanes=1 --config path100m --reps 3 --steps 2 > gpurun_out/ab_g1_path.jsonl 2>&1
grep -h lib gpurun_out/ab_g1_path.jsonl || tail -5 gpurun_out/ab_g1_path.jsonl
timeout 600 python scripts/ab_libs.py --libs $L --variant walker_lanes=32 --variant walker_lanes=1 --config road24m --reps 3 --steps 4 > gpurun_out/ab_g1_road.jsonl 2>&1
grep -h lib gpurun_out/ab_g1_road.jsonl || tail -5 gpurun_out/ab_g1_road.jsonl
