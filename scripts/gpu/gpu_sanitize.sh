cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/san
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 300 -p no:cacheprovider -x -k "fault or concurrent or one_level" > gpurun_out/san/tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/san/tests.log; tail -3 gpurun_out/san/tests.log
cat > /tmp/san_small.py <<'PY'
import sys; sys.path.insert(0, '.')
import numpy as np, graphgen, oracle
from paper_conf_ppopp_niul0c26_b200 import Graph, Options
for g in (graphgen.road(120, 90, seed=3), graphgen.rmat(12, 8, seed=5), graphgen.caterpillar(300, 20)):
    with Graph(g.row_ptr, g.col_idx) as G:
        for o in (Options(hot_cutoff=1, cold_cutoff=1, blocks=8, warps_per_block=8), Options(deterministic=True),
                  Options(ring_cap=2, blocks=4, warps_per_block=4), Options(concurrency=2, blocks=4, warps_per_block=4)):
            if o.concurrency:
                out = G.run_batch([0, 1], options=o)
                ps = [out[0].cpu().numpy(), out[1].cpu().numpy()]; rs = [0, 1]
            else:
                ps = [G.run(0, options=o).cpu().numpy()]; rs = [0]
            for p, r in zip(ps, rs):
                res = oracle.check_tree(g.row_ptr, g.col_idx, r, p)
                assert res.ok, res
print("sanitizer workload ok")
PY
for tool in memcheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python /tmp/san_small.py > gpurun_out/san/$tool.log 2>&1; echo "$tool rc=$?" | tee -a gpurun_out/san/summary.txt
  tail -4 gpurun_out/san/$tool.log
done
