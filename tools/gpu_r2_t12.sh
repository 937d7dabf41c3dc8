cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_shard.py tests/test_gpu_dist.py tests/test_gpu_bench.py -k "p2p or shard or dist or c5_line" -q --timeout 600 -p no:cacheprovider > gpurun_out/r2_t12.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t12.log
