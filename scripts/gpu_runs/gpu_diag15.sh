cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r01
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests15.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests15.log
tail -3 gpurun_out/gpu_tests15.log
for c in road24m rmat24 path100m; do
timeout 900 python bench.py --config $c --steps 6 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/b15_$c.json 2>/dev/null
python -c "import json; d=json.load(open('gpurun_out/b15_$c.json')); print(d['config']['workload'], d['value'], d['ms_per_dfs'], d['roofline']['frac'])"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dfs_persistent -s 2 -c 1 -o gpurun_out/r01/prof_rmat24_b python bench.py --config rmat24 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-validate > gpurun_out/r01/ncu_full_rmat_b.log 2>&1
