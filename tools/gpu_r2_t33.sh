cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py -q --timeout 900 -p no:cacheprovider -k "sre or c2 or c4 or full_size or dense or rounds" > gpurun_out/r2_t33.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t33.log
GSPEC_STAMPS=1 python tools/timeline.py c2 > gpurun_out/r2_t33_tl_c2.log 2>&1
for i in 1 2; do timeout 600 python bench.py --steps 50 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t33_c2.jsonl; done
timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t33_c2.jsonl
