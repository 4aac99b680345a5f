# vertex-numbering experiment on road24m (scripts/reorder_ab.py)
set -x
timeout 1500 python scripts/reorder_ab.py --config road24m --orders orig dfs0 rcm bfs0 --roots 8 --reps 3 > gpurun_out/reorder_road.jsonl 2> gpurun_out/reorder_road.err; echo rc=$?
cat gpurun_out/reorder_road.jsonl; tail -3 gpurun_out/reorder_road.err
timeout 900 python scripts/reorder_ab.py --config road24m --orders orig rcm --roots 1 --reps 1 --set deterministic=1 --validate 0 > gpurun_out/reorder_road_det.jsonl 2>&1; echo rc=$?
grep order gpurun_out/reorder_road_det.jsonl
