cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
for c in c3 c4 c1; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spec_tma -s 2 -c 1 -o gpurun_out/prof_spec2 python tools/profile_spec.py c2 sre 3 > gpurun_out/ncu_spec.log 2>&1
