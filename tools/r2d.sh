cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -k "c1_full or workload or near_ties or lattice or cell_split or dbscan or every_row or single_pass or dense_cell or grid_structure" > gpurun_out/r2d_pytest.txt 2>&1
echo "PYTEST: $(tail -1 gpurun_out/r2d_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/r2d_pytest.txt | head -8
VARS="base cur v2" REPS=3 WLS="C2-eps0.45 C5-eps0.5 C2-eps1.40 C2-eps0.15" bash tools/ab.sh 2>&1 | tee gpurun_out/r2d_ab.txt
