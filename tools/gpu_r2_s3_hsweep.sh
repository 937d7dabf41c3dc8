cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
: > gpurun_out/hs.log
for h in 0 520 600 660; do
  if [ $h = 0 ]; then timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/hs_$h.log 2>&1
  else GSPEC_DELTA_H=$h timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/hs_$h.log 2>&1; fi
  echo "H=$h $(grep -o '"value": [0-9.]*, "unit"\|"ms_per_step": [0-9.]*\|"frac": [0-9.]*' gpurun_out/hs_$h.log | head -3 | tr '\n' ' ')" >> gpurun_out/hs.log
done
for c in c2 c3; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/hs_$c.log 2>&1; echo "$c $(grep -o '"value": [0-9.]*, "unit"\|"ms_per_step": [0-9.]*\|"frac": [0-9.]*' gpurun_out/hs_$c.log | head -3 | tr '\n' ' ')" >> gpurun_out/hs.log; done
python - >> gpurun_out/hs.log 2>&1 <<'PY'
import sys; sys.path.insert(0,'.')
import torch, gen, paper_conf_ipps_wangwqw22_b200 as gs
w = gen.workload('c4'); prof = torch.empty(1<<20, dtype=torch.uint8, device='cuda'); w.device(prof, offset=w.length)
f = gs.FSM.load(w.table, w.start, w.accept, profile=prof.cpu().numpy())
t = f.transform(); print("transform", t["mode"], t["hot_rows"])
PY
