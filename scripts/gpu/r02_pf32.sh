# 32-wide step: row_ptr prefetch lanes for candidates (8 default, 2, 0)
for c in road24m grid256 path100m; do
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/pf32_2/libdfs.so ab/pf32_0/libdfs.so --config $c --reps 3 --steps 6 \
  --variant "walker_lanes=32" > gpurun_out/ab_pf32_$c.jsonl 2>&1
grep lib gpurun_out/ab_pf32_$c.jsonl || tail -20 gpurun_out/ab_pf32_$c.jsonl
done
