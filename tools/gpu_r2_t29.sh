cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py tests/test_gpu_batch.py -q --timeout 900 -p no:cacheprovider -k "c3 or batch or multi or classed" > gpurun_out/r2_t29.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t29.log
for p in 1 0; do for c in c3 c3s; do GSPEC_U16H_PAD=$p timeout 600 python bench.py --config $c --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 > gpurun_out/r2_t29_${c}_pad$p.log; done; done
