# Round 2: compute-sanitizer on the new paths (RR/NF dense rounds, faithful PM, paper-literal RR/NF,
# lookback > 2, CSE 16, ENUM 64, failed/poison shard maps, async steps, fused round 0)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
K="dense_recovery and (rr or nf) or pm_tree or literal_rr_nf or lookback_long and sre or cse_spec16 or enum_bound or vr_others"
timeout 2400 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "$K" > gpurun_out/r02_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02_memcheck.log
timeout 1800 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_shard.py -q -p no:cacheprovider -x -k "invalid_symbol_in or failed or nonmerging or async" > gpurun_out/r02_memcheck_shard.log 2>&1; echo "rc=$?" >> gpurun_out/r02_memcheck_shard.log
timeout 2400 compute-sanitizer --tool racecheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "literal_rr_nf and (c3 or rand) or pm_tree and c3 or dense_recovery and rr and 33554432" > gpurun_out/r02_racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02_racecheck.log
GSPEC_V0=1 timeout 1800 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "inline_round0" > gpurun_out/r02_memcheck_v0.log 2>&1; echo "rc=$?" >> gpurun_out/r02_memcheck_v0.log
GSPEC_V0=1 timeout 1800 compute-sanitizer --tool racecheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "inline_round0 and c2" > gpurun_out/r02_racecheck_v0.log 2>&1; echo "rc=$?" >> gpurun_out/r02_racecheck_v0.log
