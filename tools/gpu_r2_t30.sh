cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "enum_four_symbol and (rand or c1-1048576)" > gpurun_out/r2_t30_memcheck_tk.log 2>&1
timeout 1500 compute-sanitizer --tool racecheck --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "enum_four_symbol and (c1-1048576 or 300001)" > gpurun_out/r2_t30_racecheck_tk.log 2>&1
timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_p2p.py -q -p no:cacheprovider -k "c2" > gpurun_out/r2_t30_memcheck_p2p.log 2>&1
