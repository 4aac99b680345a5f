# sequential-descent L2 prefetch in the 32-wide step (ab/seqpf4) vs default; caterpillar, road, grid
for c in caterpillar road24m grid256; do
timeout 900 python scripts/ab_libs.py --libs paper_conf_ppopp_niul0c26_b200/libdfs.so ab/seqpf4/libdfs.so --config $c --reps 3 --steps 3 \
  --variant "" --variant "window=128" > gpurun_out/ab_seqpf_$c.jsonl 2>&1
grep lib gpurun_out/ab_seqpf_$c.jsonl || tail -20 gpurun_out/ab_seqpf_$c.jsonl
done
