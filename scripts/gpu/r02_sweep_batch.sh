# C5 batch: concurrency / walker / scheduling sweep (64 roots per rep, library defaults otherwise)
L=paper_conf_ppopp_niul0c26_b200/libdfs.so
timeout 1500 python scripts/ab_libs.py --libs $L --config road24m --reps 2 --batch 64 \
  --variant "" --variant "concurrency=6" --variant "concurrency=10" --variant "concurrency=12" --variant "concurrency=16" \
  --variant "steal_period=8" --variant "steal_period=32" --variant "steal_period=64" \
  --variant "hot_cutoff=2" --variant "cold_cutoff=4" --variant "donate=0" --variant "spill_idle=128" \
  --variant "backoff_max_ns=8192" --variant "walker_lanes=8,concurrency=12" > gpurun_out/sweep_batch.jsonl 2>&1
grep lib gpurun_out/sweep_batch.jsonl || tail -20 gpurun_out/sweep_batch.jsonl
