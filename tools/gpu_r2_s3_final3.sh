# Session-3 last capture (after the ENUM packed maps): same commands as gpu_r2_s3_final.sh
# launch lists (C2, C3, C3 RR), ncu --set full of C4's one-exception spec kernel and of C3's pass 0.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider --durations=10 > gpurun_out/s3z_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/s3z_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s3z_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/s3z_smoke.log
timeout 1200 python bench.py > gpurun_out/s3z_bench_default.log 2>&1
timeout 600 python bench.py --impl reference > gpurun_out/s3z_bench_reference.log 2>&1
for c in c1 c3 c3s c4; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 1 --no-per-dfa > gpurun_out/s3z_bench_$c.log 2>&1
done
for s in rr nf; do
  timeout 900 python bench.py --config c3 --scheme $s --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/s3z_bench_c3_$s.log 2>&1
done
timeout 900 python bench.py --config c3s --scheme nf --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/s3z_bench_c3s_nf.log 2>&1
timeout 1500 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/s3z_bench_c5.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s3z_launches_c2.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/s3z_ncu_launch.log 2>&1
CK_PROFILE_LAST=1 timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/s3z_launches_c3.csv python tools/ck_probe.py c3 sre 3 > gpurun_out/s3z_ncu_c3.log 2>&1
CK_PROFILE_LAST=1 timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s3z_launches_c3_rr.csv python tools/ck_probe.py c3 rr 3 > gpurun_out/s3z_ncu_c3_rr.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 60 --csv --log-file gpurun_out/s3z_launches_c4.csv python tools/profile_spec.py c4 sre 2 > gpurun_out/s3z_ncu_launch_c4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi6ELi1E -s 1 -c 1 -o /tmp/s3z_spec_c4 -f python tools/profile_spec.py c4 sre 3 > gpurun_out/s3z_ncu_c4.log 2>&1
ncu -i /tmp/s3z_spec_c4.ncu-rep --page raw --csv > gpurun_out/s3z_spec_c4_raw.csv 2>&1
