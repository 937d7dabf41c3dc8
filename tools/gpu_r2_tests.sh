# Round 2: the new GPU tests (C5 16 GiB, shard robustness, selector, vr_others) then the whole GPU suite.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_c5.py tests/test_gpu_shard.py tests/test_gpu_dist.py -q --timeout 1200 -p no:cacheprovider -k "c5 or invalid_symbol_in or failed or nonmerging or collective" --durations=10 > gpurun_out/r2_new_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2_new_tests.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 600 -p no:cacheprovider -k "enum_bound or input_sensitive or vr_others" > gpurun_out/r2_new_parity.log 2>&1; echo "rc=$?" >> gpurun_out/r2_new_parity.log
