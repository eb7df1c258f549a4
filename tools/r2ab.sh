cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:"k_ps_scatter|k_ps_hist" -c 4 -o gpurun_out/r2ab_prof_sort python bench.py --workload C5-eps0.5 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out | grep r2ab
