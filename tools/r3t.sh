cd $GRAFT_REPO_ROOT
HDB_LIB=ab/libhdb_vc3.so timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "c1_full or workload_subsets or sparse_dense or near_ties or lattice or decimal or edge_cases or dense_cell or bands_assemble or single_pass or cell_split or batching or exact_f64 or full_size_sampled" > gpurun_out/r3t_pytest.txt 2>&1
WLS="C5-eps0.5 C2-eps0.15 C2-eps0.45 C3-eps0.20" VARS="vc0 vc3" REPS=2 bash tools/ab.sh > gpurun_out/r3t_ab.txt 2>&1
