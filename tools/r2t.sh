cd $GRAFT_REPO_ROOT
HDB_LIB=ab/libhdb_sc16.so timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -k "c1_full or workload or grid_structure or every_row and C3 or shard" > gpurun_out/r2t_pytest.txt 2>&1
echo "PYTEST sc16: $(tail -1 gpurun_out/r2t_pytest.txt)"
VARS="sc8 sc16 sc4" REPS=2 WLS="C5-eps0.5 C3-eps0.07" bash tools/ab.sh 2>&1 | tee gpurun_out/r2t_ab.txt
for v in sc8 sc16; do ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2t_launches_$v.csv env HDB_LIB=ab/libhdb_$v.so python bench.py --workload C5-eps0.5 --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1; done
