# double-buffered host rows for concurrent batches: capi batch tests + the batch1024 line (e2e)
set -x
timeout 900 python -m pytest tests/test_gpu_capi_batch.py -q -x --timeout 600 > gpurun_out/pytest_e2e.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_e2e.log
timeout 900 python bench.py --config batch1024 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_batch_e2e.json 2> gpurun_out/bench_batch_e2e.err; echo bench rc=$?
tail -2 gpurun_out/bench_batch_e2e.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_batch_e2e.json').read().strip().splitlines()[-1]); print(d['value'], d.get('e2e'))"
