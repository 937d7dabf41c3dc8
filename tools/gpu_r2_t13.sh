cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
out=gpurun_out/r2_t13_sweep.jsonl; : > $out
for cfg in c3 c3s c4 c2; do for B in 1024 2048 4096 8192; do for s in auto rr nf; do
  if [ $cfg != c3 ] && [ $s != auto ]; then continue; fi
  r=$(timeout 300 python bench.py --config $cfg --scheme $s --chunk-bytes $B --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1)
  echo "{\"cfg\":\"$cfg\",\"B\":$B,\"scheme\":\"$s\",\"line\":$r}" >> $out
done; done; done
