cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py -q --timeout 900 -p no:cacheprovider -k "dense or conv_fractions or true_walk" > gpurun_out/r2_t15.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t15.log
out=gpurun_out/r2_t15_bench.jsonl; : > $out
for s in rr nf sre; do
  r=$(timeout 300 python bench.py --config c3 --scheme $s --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1)
  echo "$r" >> $out
  r=$(timeout 300 python bench.py --config c3s --scheme $s --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1)
  echo "$r" >> $out
done
