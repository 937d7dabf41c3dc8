# Targeted ncu --set full captures (mangled-name filters: the selector's sample runs and the
# spare dense-round slots launch small or early-returning instances of the same kernels)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi1ELi1ELi3ELb0ELb0E -s 1 -c 1 -o /tmp/q_spec_c2 -f python tools/profile_spec.py c2 sre 3 > gpurun_out/q_ncu_spec_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_verify_recoverILi1E -s 6 -c 1 -o /tmp/q_verify_c2 -f python tools/profile_spec.py c2 sre 3 > gpurun_out/q_ncu_verify_c2.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi4ELi1ELi2ELb0ELb0E -s 1 -c 1 -o /tmp/q_spec_c4 -f python tools/profile_spec.py c4 sre 3 > gpurun_out/q_ncu_spec_c4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi3ELi1ELi3ELb0ELb0E -s 1 -c 1 -o /tmp/q_spec_c3 -f python tools/profile_spec.py c3 sre 3 > gpurun_out/q_ncu_spec_c3.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,launch__grid_size --clock-control none --kernel-name-base mangled -k regex:k_spec_tmaILi3ELi1ELi3ELb1E --csv python tools/profile_spec.py c3 sre 4 > gpurun_out/q_task_c3_list.csv 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name-base mangled -k regex:k_spec_tmaILi1ELi1ELi3ELb0ELb0E --csv python tools/profile_spec.py c2 sre 3 > gpurun_out/q_dram_c2.csv 2>&1
for r in q_spec_c2 q_verify_c2 q_spec_c4 q_spec_c3; do
  if [ -f /tmp/$r.ncu-rep ]; then
    ncu -i /tmp/$r.ncu-rep --page raw --csv > gpurun_out/${r}_raw.csv 2>&1
    ncu -i /tmp/$r.ncu-rep --page details --csv > gpurun_out/${r}_details.csv 2>&1
  fi
done
timeout 600 python -m pytest tests/test_gpu_shard.py tests/test_gpu_c5.py tests/test_gpu_parity.py -q --timeout 900 -p no:cacheprovider -k "async or c5 or lookback_long" --durations=6 > gpurun_out/r2_t8.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t8.log
timeout 600 python bench.py --config c2 --lookback 8 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_c2_lb8.log 2>&1
du -sh gpurun_out
