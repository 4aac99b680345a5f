# thread walkers with 32-entry rings (24 warps): stats vs G=4, batch A/B
set -x
timeout 600 python scripts/walker_stats.py --config road24m --lanes 4 1 --blocks 18 > gpurun_out/g1_stats.jsonl 2>&1; echo rc=$?
cat gpurun_out/g1_stats.jsonl | tail -8
L=paper_conf_ppopp_niul0c26_b200/libdfs.so
timeout 600 python scripts/ab_libs.py --libs $L --variant walker_lanes=4 --variant walker_lanes=1 --config road24m --batch 64 --reps 3 > gpurun_out/ab_g1b_batch.jsonl 2>&1
grep -h lib gpurun_out/ab_g1b_batch.jsonl || tail -5 gpurun_out/ab_g1b_batch.jsonl
