cd $GRAFT_REPO_ROOT
VARS="prev2 spf2" REPS=2 WLS="C3-eps0.07 C3-eps0.12 C3L-eps0.07 C3L-eps0.12" bash tools/ab.sh 2>&1 | tee gpurun_out/r2z_ab.txt
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2z_launches_C3.csv env HDB_LIB=ab/libhdb_spf2.so python bench.py --workload C3-eps0.07 --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
