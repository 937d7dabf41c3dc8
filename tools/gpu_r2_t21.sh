cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -q --timeout 900 -p no:cacheprovider -k "enum or c1 or div7 or random_dfas" > gpurun_out/r2_t21.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t21.log
GSPEC_TK=1 timeout 900 python bench.py --config c5 --c5-dfa c1 --steps 5 --warmup 3 2>&1 | tail -1 > gpurun_out/r2_t21_c5c1.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r2_t21_launch_c1.csv python bench.py --config c5 --c5-dfa c1 --steps 1 --warmup 3 > /dev/null 2>&1
