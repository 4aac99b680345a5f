# walker kernel register budget: 1024-thread CTAs (64 regs, default) vs 768 (80 regs) vs 512 (96 regs)
timeout 1500 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/lb768/libdfs.so --config road24m --reps 3 --batch 128 \
  --variant "warps_per_block=24" > gpurun_out/ab_lb768_batch.jsonl 2>&1
grep lib gpurun_out/ab_lb768_batch.jsonl || tail -20 gpurun_out/ab_lb768_batch.jsonl
timeout 1500 python scripts/ab_libs.py --libs ab/lb512/libdfs.so --config road24m --reps 3 --batch 128 \
  --variant "warps_per_block=16" > gpurun_out/ab_lb512_batch.jsonl 2>&1
grep lib gpurun_out/ab_lb512_batch.jsonl || tail -20 gpurun_out/ab_lb512_batch.jsonl
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/lb768/libdfs.so --config path100m --reps 3 --steps 4 \
  --variant "warps_per_block=24" > gpurun_out/ab_lb_path.jsonl 2>&1
grep lib gpurun_out/ab_lb_path.jsonl || tail -20 gpurun_out/ab_lb_path.jsonl
