# A/B: adaptive tail speculation in the 128-wide step (spec_tail) vs the build without it
timeout 900 python scripts/ab_libs.py --libs ab/head/libdfs.so ab/spectail/libdfs.so --config rmat24 --reps 5 --steps 6 \
  --variant "" --variant "spec_tail=2" --variant "spec_tail=8" > gpurun_out/ab_spectail_rmat.jsonl 2>&1
grep lib gpurun_out/ab_spectail_rmat.jsonl || tail -20 gpurun_out/ab_spectail_rmat.jsonl
timeout 600 python scripts/ab_libs.py --libs ab/head/libdfs.so ab/spectail/libdfs.so --config road24m --reps 3 --steps 6 > gpurun_out/ab_spectail_road.jsonl 2>&1
grep lib gpurun_out/ab_spectail_road.jsonl || tail -20 gpurun_out/ab_spectail_road.jsonl
