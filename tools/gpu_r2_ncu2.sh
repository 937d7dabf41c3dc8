cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import os; print('affinity', len(os.sched_getaffinity(0)), 'cpu_count', os.cpu_count())" > gpurun_out/q_cpu.txt 2>&1
cat /sys/fs/cgroup/cpu.max >> gpurun_out/q_cpu.txt 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi5ELi1ELi2ELb0ELb0E -s 1 -c 1 -o /tmp/q_spec_c4 -f python tools/profile_spec.py c4 sre 3 > gpurun_out/q_ncu_spec_c4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi4ELi1ELi3ELb0ELb0E -s 1 -c 1 -o /tmp/q_spec_c3 -f python tools/profile_spec.py c3 sre 3 > gpurun_out/q_ncu_spec_c3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi4ELi1ELi3ELb1ELb0E -s 6 -c 1 -o /tmp/q_task_c3 -f python tools/profile_spec.py c3 sre 4 > gpurun_out/q_ncu_task_c3.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name-base mangled -k regex:k_spec_tmaILi5ELi1ELi2ELb0ELb0E --csv python tools/profile_spec.py c4 sre 3 > gpurun_out/q_dram_c4.csv 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,launch__grid_size --clock-control none --kernel-name-base mangled -k regex:k_spec_tmaILi4ELi1ELi3ELb1E --csv python tools/profile_spec.py c3 sre 4 > gpurun_out/q_task_c3_list.csv 2>&1
for r in q_spec_c4 q_spec_c3 q_task_c3; do
  if [ -f /tmp/$r.ncu-rep ]; then
    ncu -i /tmp/$r.ncu-rep --page raw --csv > gpurun_out/${r}_raw.csv 2>&1
    ncu -i /tmp/$r.ncu-rep --page details --csv > gpurun_out/${r}_details.csv 2>&1
  fi
done
