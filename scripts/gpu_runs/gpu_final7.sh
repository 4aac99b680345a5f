cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r01h
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider > gpurun_out/r01h/gpu_tests_full.log 2>&1; echo "tests rc=$?" >> gpurun_out/r01h/gpu_tests_full.log
tail -3 gpurun_out/r01h/gpu_tests_full.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01h/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r01h/smoke.log; tail -2 gpurun_out/r01h/smoke.log
timeout 900 python bench.py > gpurun_out/r01h/bench_default.json 2> gpurun_out/r01h/bench_default.err; echo "default bench rc=$?"
head -c 600 gpurun_out/r01h/bench_default.json; echo
timeout 900 python bench.py --config batch1024 --warmup 3 > gpurun_out/r01h/bench_batch1024.json 2> gpurun_out/r01h/bench_batch1024.err
python -c "import json; d=json.load(open('gpurun_out/r01h/bench_batch1024.json')); print('batch1024', d['value'], d['dfs_per_s'], d['concurrency'])"
