cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_shard.py -q -x -k "nccl or fake_collective" --timeout 900 -p no:cacheprovider > gpurun_out/pytest_shard.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_shard.log
timeout 900 compute-sanitizer --tool racecheck --print-limit 10 python tools/profile_spec.py c3 sre 1 > gpurun_out/racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/racecheck.log
timeout 900 compute-sanitizer --tool synccheck --print-limit 10 python -m pytest tests/test_gpu_parity.py -q -x -k "random_dfas and (1 or 2)" -p no:cacheprovider > gpurun_out/synccheck.log 2>&1; echo "rc=$?" >> gpurun_out/synccheck.log
