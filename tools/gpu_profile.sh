# Round profile capture: GPU tests, default bench line, every config's bench line, ncu launch
# list of the bench command, ncu --set full of the kernels of a run (c2 spec + verify, c4 spec),
# batch throughput.  Usage (from gpurun):  bash tools/gpu_profile.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider > gpurun_out/pytest_gpu_all.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_all.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1
for c in c1 c3 c3s c4; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 1 > gpurun_out/bench_$c.log 2>&1
done
GSPEC_STAMPS=1 timeout 600 python tools/timeline.py c2 > gpurun_out/timeline_c2.log 2>&1
GSPEC_STAMPS=1 timeout 600 python tools/timeline.py c4 > gpurun_out/timeline_c4.log 2>&1
timeout 900 python tools/bench_batch.py c2 c3 c4 > gpurun_out/bench_batch.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spec_tma -s 2 -c 1 -o gpurun_out/spec_tma_c2 -f python tools/profile_spec.py c2 sre 3 > gpurun_out/ncu_spec.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_verify_recover -s 2 -c 1 -o gpurun_out/verify_c2 -f python tools/profile_spec.py c2 sre 3 > gpurun_out/ncu_verify.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_spec_tma -s 2 -c 1 -o gpurun_out/spec_tma_c4 -f python tools/profile_spec.py c4 sre 3 > gpurun_out/ncu_spec_c4.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_c3.csv python tools/profile_spec.py c3 sre 2 > gpurun_out/ncu_launch_c3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spec_tma -s 1 -c 1 -o gpurun_out/task_gather_c3 -f python tools/profile_spec.py c3 sre 1 > gpurun_out/ncu_task_c3.log 2>&1
for c in c1 c2 c3 c4; do
  timeout 600 python bench.py --config $c --scheme cse --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_cse_$c.log 2>&1
done
