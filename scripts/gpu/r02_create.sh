# dfs_graph_create from pageable host memory: bounce-buffer upload (default) vs plain cudaMemcpy (ab/head)
for rep in 1 2; do
for lib in ab/head/libdfs.so paper_conf_ppopp_niul0c26_b200/libdfs.so; do
DFS_LIB=$lib timeout 600 python scripts/create_timing.py road24m 4 pageable,pinned >> gpurun_out/create_ab.jsonl 2>&1
done
done
cat gpurun_out/create_ab.jsonl | grep create_ms
