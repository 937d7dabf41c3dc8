# compute-sanitizer over the paths added late this session: paper-literal kernel, chained
# verification passes, device-driven dense rounds, speculative shard maps (fake collective).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1500 $CS --tool memcheck python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py -q -x -p no:cacheprovider -k "literal or chained or dense or (fake_collective and (c1 or c3) and 2)" > gpurun_out/memcheck2.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/memcheck2.log
timeout 1500 $CS --tool racecheck python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "literal or (chained and cse-64)" > gpurun_out/racecheck2.log 2>&1; echo "racecheck rc=$?" >> gpurun_out/racecheck2.log
timeout 1500 $CS --tool synccheck python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "literal or (chained and cse-64)" > gpurun_out/synccheck2.log 2>&1; echo "synccheck rc=$?" >> gpurun_out/synccheck2.log
