cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_c5.py tests/test_gpu_shard.py -m gpu -q --timeout 1200 -p no:cacheprovider -x -k "c1 or enum or div7" > gpurun_out/pk_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pk_pytest.log
: > gpurun_out/pk.log
timeout 900 python bench.py --config c5 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/pk_c5.log 2>&1
GSPEC_TK_PK=0 timeout 900 python bench.py --config c5 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/pk0_c5.log 2>&1
timeout 600 python bench.py --config c1 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/pk_c1.log 2>&1
python - >> gpurun_out/pk.log <<'PY'
import json
for f in ('gpurun_out/pk_c5.log','gpurun_out/pk0_c5.log','gpurun_out/pk_c1.log'):
    for l in open(f):
        if l.startswith('{'):
            d=json.loads(l)
            print(f, d['value'], d['ms_per_step'], {k: (v.get('value'), v.get('ms_per_step')) for k, v in (d.get('per_dfa') or {}).items()} if isinstance(d.get('per_dfa'), dict) else '')
PY
