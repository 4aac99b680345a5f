# warp kernel CTA: 32 warps x 64 registers (default) vs 28 x 72 (ab/w28, no spills in the 128-wide step)
for c in road24m rmat24 grid256; do
timeout 1200 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/w28/libdfs.so --config $c --reps 5 --steps 6 > gpurun_out/ab_w28_$c.jsonl 2>&1
grep -h lib gpurun_out/ab_w28_$c.jsonl || tail -5 gpurun_out/ab_w28_$c.jsonl
done
timeout 1200 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/w28/libdfs.so --config caterpillar --reps 3 --steps 2 > gpurun_out/ab_w28_caterpillar.jsonl 2>&1
grep -h lib gpurun_out/ab_w28_caterpillar.jsonl
# walker default now 28 warps: batch + path vs the 32-warp walker (explicit warps_per_block=32 clamps to 28 -> use old build ab/wpf0)
timeout 1200 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/wpf0/libdfs.so --config road24m --reps 3 --batch 128 > gpurun_out/ab_w28_batch.jsonl 2>&1
grep -h lib gpurun_out/ab_w28_batch.jsonl
