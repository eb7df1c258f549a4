cd $GRAFT_REPO_ROOT
HDB_TRACE=1 timeout 300 python bench.py --workload C3-eps0.07 --steps 3 --warmup 2 --e2e-steps 0 --no-cpu-baseline > /dev/null 2> gpurun_out/r2x_trace_C3.txt
HDB_TRACE=1 timeout 300 python bench.py --workload C2-eps0.45 --steps 3 --warmup 2 --e2e-steps 0 --no-cpu-baseline > /dev/null 2> gpurun_out/r2x_trace_C2.txt
HDB_TRACE=1 timeout 300 python bench.py --workload C1-eps0.5 --steps 3 --warmup 2 --e2e-steps 0 --no-cpu-baseline > /dev/null 2> gpurun_out/r2x_trace_C1.txt
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2x_launches_C3.csv python bench.py --workload C3-eps0.07 --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
