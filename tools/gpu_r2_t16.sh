cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py tests/test_gpu_batch.py -q --timeout 900 -p no:cacheprovider -k "c4 or delta or classed or batch or multi" > gpurun_out/r2_t16.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t16.log
for i in 1 2; do timeout 300 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t16_bench.jsonl; done
