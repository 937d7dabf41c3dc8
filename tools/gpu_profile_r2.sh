# Round-2 capture: full GPU tests, smoke, the default bench line (+ per-DFA sub-results), the C5
# line on one GPU, every config / scheme line, ncu launch lists and --set full captures of the
# dominant kernels, the experiment analogues and the literal-vs-pipeline comparison.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider --durations=15 > gpurun_out/p2_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/p2_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/p2_smoke.log 2>&1
timeout 1200 python bench.py > gpurun_out/p2_bench_default.log 2>&1
timeout 1500 python bench.py --config c5 --steps 5 --warmup 3 > gpurun_out/p2_bench_c5.log 2>&1
for c in c1 c3 c3s c4; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 1 --no-per-dfa > gpurun_out/p2_bench_$c.log 2>&1
done
for s in rr nf pm cse; do
  timeout 900 python bench.py --config c3 --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/p2_bench_c3_$s.log 2>&1
done
timeout 900 python bench.py --config c3 --scheme cse --spec-k 16 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/p2_bench_c3_cse16.log 2>&1
timeout 900 python bench.py --config c2 --scheme pm_tree --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/p2_bench_c2_pmtree.log 2>&1
timeout 900 python bench.py --config c2 --lookback 8 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/p2_bench_c2_lb8.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/p2_launches_c2.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/p2_ncu_launch.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/p2_launches_c3.csv python tools/profile_spec.py c3 sre 2 > gpurun_out/p2_ncu_launch_c3.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/p2_launches_c3_rr.csv python tools/profile_spec.py c3 rr 2 > gpurun_out/p2_ncu_launch_c3_rr.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spec_tma -s 2 -c 1 -o /tmp/p2_spec_tma_c2 -f python tools/profile_spec.py c2 sre 3 > gpurun_out/p2_ncu_spec.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_verify_recover -s 2 -c 1 -o /tmp/p2_verify_c2 -f python tools/profile_spec.py c2 sre 3 > gpurun_out/p2_ncu_verify.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_spec_tma -s 2 -c 1 -o /tmp/p2_spec_tma_c4 -f python tools/profile_spec.py c4 sre 3 > gpurun_out/p2_ncu_spec_c4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spec_tma -s 1 -c 1 -o /tmp/p2_task_gather_c3 -f python tools/profile_spec.py c3 sre 1 > gpurun_out/p2_ncu_task_c3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_verify_recover -s 0 -c 1 -o /tmp/p2_verify_c3_rr -f python tools/profile_spec.py c3 rr 1 > gpurun_out/p2_ncu_verify_rr.log 2>&1
timeout 1500 python tools/experiments.py --mib 64 --reps 2 --out gpurun_out/p2_experiments.md > gpurun_out/p2_experiments.log 2>&1
timeout 600 python tools/literal_vs_pipeline.py > gpurun_out/p2_lit_vs_pipe.jsonl 2>&1
for r in p2_spec_tma_c2 p2_verify_c2 p2_spec_tma_c4 p2_task_gather_c3 p2_verify_c3_rr; do
  if [ -f /tmp/$r.ncu-rep ]; then
    ncu -i /tmp/$r.ncu-rep --page raw --csv > gpurun_out/${r}_raw.csv 2>&1
    ncu -i /tmp/$r.ncu-rep --page details --csv > gpurun_out/${r}_details.csv 2>&1
    ncu -i /tmp/$r.ncu-rep --page source --csv --print-source sass > /tmp/${r}_src.csv 2>&1; head -c 4000000 /tmp/${r}_src.csv > gpurun_out/${r}_source_head.csv
  fi
done
du -sh gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py -q --timeout 900 -p no:cacheprovider -k "enum_bound or random_dfas or div7_c1 or nonmerging or fake_collective" > gpurun_out/r2_t7.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t7.log
for e in 0 1; do for p in 0 1; do
  GSPEC_TMA_EVICT=$e GSPEC_TMA_PROMO=$p timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_tma_c4_e${e}p${p}.log 2>&1
  GSPEC_TMA_EVICT=$e GSPEC_TMA_PROMO=$p timeout 600 python bench.py --config c2 --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_tma_c2_e${e}p${p}.log 2>&1
done; done
GSPEC_TMA_EVICT=1 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_spec_tma -s 2 -c 1 --csv python tools/profile_spec.py c4 sre 3 > gpurun_out/r2_tma_c4_evictnormal_dram.csv 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_spec_tma -s 2 -c 1 --csv python tools/profile_spec.py c4 sre 3 > gpurun_out/r2_tma_c4_default_dram.csv 2>&1
