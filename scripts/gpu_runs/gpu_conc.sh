cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x > gpurun_out/gpu_tests16.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests16.log
tail -3 gpurun_out/gpu_tests16.log
for c in 1 2 3 4 6; do
timeout 600 python bench.py --config batch1024 --batch-roots 256 --warmup 3 --concurrency $c > gpurun_out/bconc_$c.json 2>gpurun_out/bconc_$c.err
python -c "import json; d=json.load(open('gpurun_out/bconc_$c.json')); print('conc', d['concurrency'], d['value'], 'GTEPS', d['dfs_per_s'], 'dfs/s', d['dfs_per_s_region'])" || tail -3 gpurun_out/bconc_$c.err
done
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 1 --steps 4 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_torchrun1.json 2> gpurun_out/bench_torchrun1.err; echo "torchrun rc=$?"; cat gpurun_out/bench_torchrun1.json | head -c 400
