cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_bench.py tests/test_gpu_shard.py -q --timeout 900 -p no:cacheprovider -k "p2p or bench_c5 or async or nccl" > gpurun_out/r2_t9.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t9.log
