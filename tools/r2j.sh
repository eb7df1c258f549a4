cd $GRAFT_REPO_ROOT
HDB_LIB=ab/libhdb_pf.so timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -k "c1_full or workload or near_ties or lattice or cell_split or C5 or C2-eps0.45" > gpurun_out/r2j_pytest.txt 2>&1
echo "PYTEST pf: $(tail -1 gpurun_out/r2j_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/r2j_pytest.txt | head -8
VARS="csel pf pfb6" REPS=2 WLS="C5-eps0.5 C2-eps0.45 C2-eps1.40 C2-eps0.15" bash tools/ab.sh 2>&1 | tee gpurun_out/r2j_ab.txt
