cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "query_lane or c1_full or workload_subsets or sparse_dense or many_hits or near_ties or lattice or decimal or edge_cases or dense_cell or bands_assemble or bands_empty or single_pass" > gpurun_out/r3e_pytest.txt 2>&1
for wl in C5-eps0.5 C2-eps0.15 C3-eps0.07 C3L-eps0.07 C1-eps0.5; do
  HDB_QLANES=1 timeout 300 python bench.py --workload $wl --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r3e_bench_${wl}.json 2> gpurun_out/r3e_bench_${wl}.err
done
ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/r3e_launches_C5.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
