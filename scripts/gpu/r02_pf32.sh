# 32-wide step: row_ptr prefetch lanes for candidates (8 default, 2, 0)
for c in road24m grid256 path100m; do
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/pf32_2/libdfs.so ab/pf32_0/libdfs.so --config $c --reps 3 --steps 6 \
  --variant "walker_lanes=32" > gpurun_out/ab_pf32_$c.jsonl 2>&1
grep lib gpurun_out/ab_pf32_$c.jsonl || tail -20 gpurun_out/ab_pf32_$c.jsonl
done
# walker kernel: candidate row_ptr prefetch (min(G, 8) lanes default) vs none
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/wpf0/libdfs.so --config road24m --reps 3 --batch 64 > gpurun_out/ab_wpf_batch.jsonl 2>&1
grep lib gpurun_out/ab_wpf_batch.jsonl || tail -20 gpurun_out/ab_wpf_batch.jsonl
timeout 600 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/wpf0/libdfs.so --config path100m --reps 3 --steps 4 > gpurun_out/ab_wpf_path.jsonl 2>&1
grep lib gpurun_out/ab_wpf_path.jsonl || tail -20 gpurun_out/ab_wpf_path.jsonl
