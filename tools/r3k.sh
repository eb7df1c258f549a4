cd $GRAFT_REPO_ROOT
for cs in 1 2 3; do
  for q in 1 0; do
    HDB_QLANES=$q timeout 300 python bench.py --cell-split $cs --steps 5 --warmup 2 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r3k_C5_k${cs}_q$q.json 2>/dev/null
  done
done
HDB_QLANES=1 timeout 300 python bench.py --workload C2-eps0.45 --steps 5 --warmup 2 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r3k_C2045_q1.json 2>/dev/null
HDB_QLANES=1 timeout 300 python bench.py --workload C2-eps1.40 --steps 5 --warmup 2 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r3k_C2140_q1.json 2>/dev/null
