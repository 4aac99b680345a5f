cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/san
timeout 2400 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 30 python /tmp/san_small.py > gpurun_out/san/racecheck.log 2>&1 || true
cat > /tmp/san_small.py <<'PY'
import sys; sys.path.insert(0, '.')
import graphgen, oracle
from paper_conf_ppopp_niul0c26_b200 import Graph, Options
g = graphgen.road(60, 50, seed=3)
with Graph(g.row_ptr, g.col_idx) as G:
    for o in (Options(hot_cutoff=1, cold_cutoff=1, blocks=2, warps_per_block=4), Options(deterministic=True)):
        p = G.run(0, options=o).cpu().numpy()
        assert oracle.check_tree(g.row_ptr, g.col_idx, 0, p).ok
print("racecheck workload ok")
PY
timeout 2400 compute-sanitizer --tool racecheck --racecheck-report analysis --print-limit 30 python /tmp/san_small.py > gpurun_out/san/racecheck.log 2>&1; echo "racecheck rc=$?"
grep -E "ERROR SUMMARY|RACECHECK SUMMARY|hazard|Race reported|workload" gpurun_out/san/racecheck.log | head -20
