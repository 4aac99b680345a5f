cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ablation
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 240 -p no:cacheprovider -x -k "one_level or concurrent or stress" > gpurun_out/gpu_tests_abl.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests_abl.log
tail -3 gpurun_out/gpu_tests_abl.log
timeout 2400 python scripts/ablation.py --graphs road:4900,rmat:22 --roots 2 --reps 2 --out gpurun_out/ablation > gpurun_out/ablation/ablation.log 2> gpurun_out/ablation/ablation.err
tail -3 gpurun_out/ablation/ablation.err
cat gpurun_out/ablation/ablation.md
