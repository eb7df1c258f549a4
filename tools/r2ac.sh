cd $GRAFT_REPO_ROOT
HDB_LIB=ab/libhdb_h2.so timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -k "workload or c1_full or band or shard or grid_structure or every_row and C5" > gpurun_out/r2ac_pytest.txt 2>&1
echo "PYTEST h2: $(tail -1 gpurun_out/r2ac_pytest.txt)"
VARS="spf2 h2" REPS=3 WLS="C5-eps0.5 C2-eps0.45" bash tools/ab.sh 2>&1 | tee gpurun_out/r2ac_ab.txt
