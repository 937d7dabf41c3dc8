cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
out=gpurun_out/r2_t17_c5sweep.jsonl; : > $out
for B in 4096 8192 16384; do
  r=$(timeout 900 python bench.py --config c5 --chunk-bytes $B --steps 5 --warmup 3 2>&1 | tail -1)
  echo "{\"B\":$B,\"line\":$r}" >> $out
done
