cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -q --timeout 900 -p no:cacheprovider -k "conv_fractions or spread_profile or dense_recovery or selector_features" > gpurun_out/r2_t14.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t14.log
out=gpurun_out/r2_t14_bench.jsonl; : > $out
for cfg in c3 c3s c4 c2; do
  r=$(timeout 300 python bench.py --config $cfg --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1)
  echo "$r" >> $out
done
for s in rr nf; do
  r=$(timeout 300 python bench.py --config c3 --scheme $s --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1)
  echo "$r" >> $out
done
