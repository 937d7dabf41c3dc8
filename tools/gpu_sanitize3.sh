# compute-sanitizer over the last additions: single-launch ENUM, FSM-level batching,
# U16H pre-multiplied codes (C3 parity), round-0 shortcut + speculative finalize (C2/C4).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1500 $CS --tool memcheck python -m pytest tests/test_gpu_parity.py tests/test_gpu_batch.py -q -x -p no:cacheprovider -k "div7 or fsm_level or (configs_small and (sre or cse))" > gpurun_out/memcheck3.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/memcheck3.log
timeout 1500 $CS --tool racecheck python -m pytest tests/test_gpu_parity.py tests/test_gpu_batch.py -q -x -p no:cacheprovider -k "(div7 and enum) or fsm_level_batching_invalid" > gpurun_out/racecheck3.log 2>&1; echo "racecheck rc=$?" >> gpurun_out/racecheck3.log
