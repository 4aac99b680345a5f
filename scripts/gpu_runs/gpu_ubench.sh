cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ubench
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubench_chain scripts/ubench_chain.cu && timeout 120 /tmp/ubench_chain > gpurun_out/ubench/chain.json 2>&1
cat gpurun_out/ubench/chain.json
