cd $GRAFT_REPO_ROOT
HDB_LIB=ab/libhdb_pi4b.so timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -k "workload or c1_full or grid_structure or deterministic or every_row and C5" > gpurun_out/r2ad_pytest.txt 2>&1
echo "PYTEST pi4b: $(tail -1 gpurun_out/r2ad_pytest.txt)"
VARS="pi8 pi4 pi4b" REPS=3 WLS="C5-eps0.5 C2-eps0.45" bash tools/ab.sh 2>&1 | tee gpurun_out/r2ad_ab.txt
