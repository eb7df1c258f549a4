cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/r3s_pytest.txt 2>&1
for wl in C5-eps0.5 C2-eps0.15 C3-eps0.07; do
  timeout 300 python bench.py --workload $wl --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r3s_bench_${wl}.json 2> gpurun_out/r3s_bench_${wl}.err
done
