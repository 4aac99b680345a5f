# knob checks: batch concurrency 7/9 around the default 8; warp-kernel CTA size 28/30 vs 32 on road
set -x
L=paper_conf_ppopp_niul0c26_b200/libdfs.so
timeout 900 python scripts/ab_libs.py --libs $L --variant "" --variant concurrency=7 --variant concurrency=9 --config road24m --batch 64 --reps 5 > gpurun_out/ab_knob_conc.jsonl 2>&1
grep -h lib gpurun_out/ab_knob_conc.jsonl || tail -5 gpurun_out/ab_knob_conc.jsonl
timeout 900 python scripts/ab_libs.py --libs $L --variant "" --variant warps_per_block=30 --variant warps_per_block=28 --config road24m --reps 5 --steps 8 > gpurun_out/ab_knob_warps.jsonl 2>&1
grep -h lib gpurun_out/ab_knob_warps.jsonl || tail -5 gpurun_out/ab_knob_warps.jsonl
