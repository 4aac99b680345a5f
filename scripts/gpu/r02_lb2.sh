# walker kernel CTA size: 20 warps (lb640), 24 (lb768), 28 (lb896)
timeout 1500 python scripts/ab_libs.py --libs ab/lb640/libdfs.so --config road24m --reps 3 --batch 128 --variant "warps_per_block=20" > gpurun_out/ab_lb640_batch.jsonl 2>&1
timeout 1500 python scripts/ab_libs.py --libs ab/lb768/libdfs.so --config road24m --reps 3 --batch 128 --variant "warps_per_block=24" > gpurun_out/ab_lb768b_batch.jsonl 2>&1
timeout 1500 python scripts/ab_libs.py --libs ab/lb896/libdfs.so --config road24m --reps 3 --batch 128 --variant "warps_per_block=28" > gpurun_out/ab_lb896_batch.jsonl 2>&1
grep -h lib gpurun_out/ab_lb640_batch.jsonl gpurun_out/ab_lb768b_batch.jsonl gpurun_out/ab_lb896_batch.jsonl
for v in "640 20" "768 24" "896 28"; do set -- $v
timeout 900 python scripts/ab_libs.py --libs ab/lb$1/libdfs.so --config path100m --reps 3 --steps 4 --variant "warps_per_block=$2" > gpurun_out/ab_lb$1_path.jsonl 2>&1
grep -h lib gpurun_out/ab_lb$1_path.jsonl
done
