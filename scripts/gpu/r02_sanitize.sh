# compute-sanitizer on the round-2 default kernels: warp kernel (32-wide BULK, 128-wide BULK),
# walker kernel (4/8/16 lanes), batches on both; every tree checked with the oracle (I1-I6)
mkdir -p gpurun_out/san
cat > /tmp/san_small.py <<'PY'
import sys; sys.path.insert(0, '.')
import graphgen, oracle
from paper_conf_ppopp_niul0c26_b200 import Graph, Options as _O
def Options(**k):
    k.setdefault('timeout_ms', 1_800_000)   # 30 min: kernels run ~100x slower under the sanitizer
    return _O(**k)
cases = (graphgen.road(120, 90, seed=3), graphgen.rmat(12, 8, seed=5), graphgen.caterpillar(300, 20),
         graphgen.path_chords(20000, 200, seed=4))
opts = [Options(blocks=8, warps_per_block=8), Options(window=128, blocks=8, warps_per_block=8),
        Options(deterministic=True), Options(ring_cap=2, blocks=4, warps_per_block=4)]
for L in (4, 8, 16):
    opts += [Options(walker_lanes=L, blocks=6, warps_per_block=4), Options(walker_lanes=L, ring_cap=3, blocks=4, warps_per_block=2),
             Options(walker_lanes=L, blocks=3, warps_per_block=4, hot_cutoff=2, cold_cutoff=2, steal_period=1)]
for g in cases:
    with Graph(g.row_ptr, g.col_idx) as G:
        for o in opts:
            p = G.run(0, options=o).cpu().numpy()
            res = oracle.check_tree(g.row_ptr, g.col_idx, 0, p)
            assert res.ok, (g.name, o, res)
        for o in (Options(concurrency=2, blocks=4, warps_per_block=4), Options(concurrency=2, blocks=4, warps_per_block=4, walker_lanes=4)):
            out = G.run_batch([0, 1], options=o)
            for q, r in enumerate((0, 1)):
                assert oracle.check_tree(g.row_ptr, g.col_idx, r, out[q].cpu().numpy()).ok
print("sanitizer workload ok")
PY
for tool in ${SAN_TOOLS:-memcheck synccheck}; do
  timeout 2400 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python /tmp/san_small.py > gpurun_out/san/$tool.log 2>&1; echo "$tool rc=$?" | tee -a gpurun_out/san/summary.txt
  tail -4 gpurun_out/san/$tool.log
done
cat > /tmp/san_race.py <<'PY'
import sys; sys.path.insert(0, '.')
import graphgen, oracle
from paper_conf_ppopp_niul0c26_b200 import Graph, Options
g = graphgen.road(60, 50, seed=3)
with Graph(g.row_ptr, g.col_idx) as G:
    for o in (Options(blocks=2, warps_per_block=4), Options(walker_lanes=4, blocks=2, warps_per_block=2),
              Options(walker_lanes=8, blocks=2, warps_per_block=2)):
        p = G.run(0, options=o).cpu().numpy()
        assert oracle.check_tree(g.row_ptr, g.col_idx, 0, p).ok
print("racecheck workload ok")
PY
[ -n "$SAN_SKIP_RACE" ] || timeout 2400 compute-sanitizer --tool racecheck --racecheck-report analysis --print-limit 40 python /tmp/san_race.py > gpurun_out/san/racecheck.log 2>&1; echo "racecheck rc=$?" | tee -a gpurun_out/san/summary.txt
grep -E "ERROR SUMMARY|RACECHECK SUMMARY|Race reported|workload" gpurun_out/san/racecheck.log | head -20
