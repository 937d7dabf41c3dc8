# Round-2 final capture (after R29): full GPU tests, smoke, default bench (+ per-DFA), C5, every
# config / scheme line, launch lists of C2 / C3 (8 KiB chunks) / C3 RR, ncu --set full of C3's spec
# kernel and dense task round at 8 KiB, memcheck of the selector's convergence kernel.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider --durations=20 > gpurun_out/f_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/f_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/f_smoke.log
timeout 1200 python bench.py > gpurun_out/f_bench_default.log 2>&1
timeout 1500 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/f_bench_c5.log 2>&1
for c in c1 c3 c3s c4; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 1 --no-per-dfa > gpurun_out/f_bench_$c.log 2>&1
done
for s in rr nf pm cse; do
  timeout 900 python bench.py --config c3 --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/f_bench_c3_$s.log 2>&1
done
timeout 900 python bench.py --config c3s --scheme nf --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/f_bench_c3s_nf.log 2>&1
timeout 900 python bench.py --config c3 --scheme cse --spec-k 16 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/f_bench_c3_cse16.log 2>&1
timeout 900 python bench.py --config c2 --scheme pm_tree --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/f_bench_c2_pmtree.log 2>&1
timeout 900 python bench.py --config c2 --lookback 8 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/f_bench_c2_lb8.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/f_launches_c2.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/f_ncu_launch.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/f_launches_c3.csv python tools/profile_spec.py c3 sre 2 > gpurun_out/f_ncu_launch_c3.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/f_launches_c3_rr.csv python tools/profile_spec.py c3 rr 2 > gpurun_out/f_ncu_launch_c3_rr.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi4ELi1ELi3ELb0ELb0E -s 1 -c 1 -o /tmp/f_spec_c3 -f python tools/profile_spec.py c3 sre 3 > gpurun_out/f_ncu_spec_c3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi4ELi1ELi3ELb1ELb0E -s 1 -c 1 -o /tmp/f_task_c3 -f python tools/profile_spec.py c3 sre 4 > gpurun_out/f_ncu_task_c3.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name-base mangled -k regex:k_spec_tmaILi4ELi1ELi3ELb0ELb0E --csv python tools/profile_spec.py c3 sre 3 > gpurun_out/f_dram_c3.csv 2>&1
for r in f_spec_c3 f_task_c3; do
  if [ -f /tmp/$r.ncu-rep ]; then
    ncu -i /tmp/$r.ncu-rep --page raw --csv > gpurun_out/${r}_raw.csv 2>&1
    ncu -i /tmp/$r.ncu-rep --page details --csv > gpurun_out/${r}_details.csv 2>&1
  fi
done
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "conv_fractions and c3" > gpurun_out/f_memcheck_conv.log 2>&1
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "dense_slots_follow" > gpurun_out/f_memcheck_dense_slots.log 2>&1
du -sh gpurun_out
