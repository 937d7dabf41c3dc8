cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_bench.py tests/test_gpu_shard.py tests/test_gpu_dist.py -q --timeout 600 -p no:cacheprovider > gpurun_out/r2_t19.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t19.log
timeout 1500 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/r2_t19_c5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi4ELi1ELi3ELb1ELb0E -s 4 -c 1 -o /tmp/f_task_c3 -f python tools/profile_spec.py c3 sre 3 > gpurun_out/r2_t19_ncu_task_c3.log 2>&1
if [ -f /tmp/f_task_c3.ncu-rep ]; then ncu -i /tmp/f_task_c3.ncu-rep --page raw --csv > gpurun_out/r2_t19_task_c3_raw.csv 2>&1; fi
