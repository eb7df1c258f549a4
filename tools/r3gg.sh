cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -x -q -k "sweep or dbscan or partition" > gpurun_out/r3gg_pytest.txt 2>&1
python tools/pos_space_check.py C5 0.5 4 > gpurun_out/r3gg_pos.txt 2>&1
python tools/pos_space_check.py C2 0.45 4 >> gpurun_out/r3gg_pos.txt 2>&1
python tools/pos_space_check.py C2 1.40 16 >> gpurun_out/r3gg_pos.txt 2>&1
python bench.py --workload C4-sweep --steps 3 --warmup 1 > gpurun_out/r3gg_bench_C4.json 2> gpurun_out/r3gg_bench_C4.err
