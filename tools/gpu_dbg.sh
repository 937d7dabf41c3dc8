cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "random_dfas and 4" -p no:cacheprovider > gpurun_out/dbg1.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "random_dfas" -p no:cacheprovider > gpurun_out/dbg2.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "test_random_dfas and (rr or nf)" -p no:cacheprovider > gpurun_out/dbg3.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q --collect-only -k "random_dfas" -p no:cacheprovider > gpurun_out/dbg4.log 2>&1
