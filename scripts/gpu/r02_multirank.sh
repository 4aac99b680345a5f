# exercise bench.py's N = 2 code paths on one GPU: two ranks share cuda:0, collectives over gloo
# (DFS_BENCH_BACKEND=gloo is a test aid; timings are meaningless: the two ranks time-slice the GPU)
DFS_BENCH_BACKEND=gloo timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --steps 4 --warmup 3 --no-rmat --cpu-seconds 2 > gpurun_out/bench_2rank.json 2> gpurun_out/bench_2rank.err; echo 2rank rc=$?
tail -5 gpurun_out/bench_2rank.err
python -c "
import json; d=json.load(open('gpurun_out/bench_2rank.json')); b=d['batch1024']
print(d['n_gpus'], d['value'], d['config']['parallelism'], d['roofline']['frac'])
print(b['roots'], b['dfs_per_s'], b.get('with_gather'), b['validation'], b.get('e2e'))
"
