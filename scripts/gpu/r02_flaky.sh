# repeat the GPU suite (minus the slow full-size/bench tests) to look for intermittent failures
set -x
for rep in 1 2 3; do
timeout 1200 python -m pytest tests -m gpu -q -rf --timeout 600 -p no:cacheprovider --deselect tests/test_bench_contract.py::test_product_arm_json_line \
  --ignore tests/test_gpu_fullsize.py > gpurun_out/pytest_rep$rep.log 2>&1; echo rep $rep rc=$?
tail -2 gpurun_out/pytest_rep$rep.log
done
timeout 900 python -m pytest tests/test_bench_contract.py tests/test_gpu_fullsize.py -q -rf --timeout 600 > gpurun_out/pytest_full.log 2>&1; echo full rc=$?
tail -3 gpurun_out/pytest_full.log
