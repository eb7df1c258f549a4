cd $GRAFT_REPO_ROOT
HDB_LIB=ab/libhdb_mo2.so timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -k "c1_full or workload or near_ties or lattice or cell_split or single_pass or every_row or shard or band" > gpurun_out/r2s_pytest.txt 2>&1
echo "PYTEST mo2: $(tail -1 gpurun_out/r2s_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/r2s_pytest.txt | head -8
VARS="base2 mo1 mo2" REPS=3 WLS="C5-eps0.5 C2-eps0.45 C3-eps0.07" bash tools/ab.sh 2>&1 | tee gpurun_out/r2s_ab.txt
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2s_launches_C5.csv env HDB_LIB=ab/libhdb_mo2.so python bench.py --workload C5-eps0.5 --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
