cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batch.py tests/test_gpu_records.py tests/test_gpu_shard.py -m gpu -q --timeout 900 -p no:cacheprovider -x -k "c4 or delta or batch or records" > gpurun_out/d1_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/d1_pytest.log
timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/d1_bench_c4.log 2>&1
GSPEC_DELTA_EXC=2 timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/d1_bench_c4_exc2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi6ELi1E -s 1 -c 1 -o /tmp/d1_spec_c4 -f python tools/profile_spec.py c4 sre 3 > gpurun_out/d1_ncu.log 2>&1
ncu -i /tmp/d1_spec_c4.ncu-rep --page raw --csv > gpurun_out/d1_spec_c4_raw.csv 2>&1
