cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r01
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests14.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests14.log
tail -3 gpurun_out/gpu_tests14.log
timeout 900 python bench.py --config batch1024 --warmup 3 > gpurun_out/bench_batch.json 2> gpurun_out/bench_batch.err; cat gpurun_out/bench_batch.json; tail -2 gpurun_out/bench_batch.err
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_road.json 2> gpurun_out/bench_road.err; cat gpurun_out/bench_road.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01/launches_road24m.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/r01/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 2 -c 1 -o gpurun_out/r01/prof_road24m python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/r01/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 2 -c 1 -o gpurun_out/r01/prof_rmat24 python bench.py --config rmat24 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/r01/ncu_full_rmat.log 2>&1
ls -la gpurun_out/r01
