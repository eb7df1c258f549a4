cd $GRAFT_REPO_ROOT
HDB_LIB=ab/libhdb_pf1.so timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -k "natural_order or C5 or shard or band or workload" > gpurun_out/r2af_pytest.txt 2>&1
echo "PYTEST pf1: $(tail -1 gpurun_out/r2af_pytest.txt)"
VARS="pf0 pf1" REPS=4 WLS="C5-eps0.5 C2-eps0.45" bash tools/ab.sh 2>&1 | tee gpurun_out/r2af_ab.txt
