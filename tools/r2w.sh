cd $GRAFT_REPO_ROOT
HDB_LIB=ab/libhdb_nc1.so timeout 1200 python -m pytest tests -m gpu -q -x --timeout 600 -k "not every_row or C5 or C3" > gpurun_out/r2w_pytest.txt 2>&1
echo "PYTEST nc1: $(tail -1 gpurun_out/r2w_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/r2w_pytest.txt | head -5
VARS="prev nc1" REPS=3 WLS="C5-eps0.5 C2-eps0.45 C3-eps0.07" bash tools/ab.sh 2>&1 | tee gpurun_out/r2w_ab.txt
