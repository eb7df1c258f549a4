cd $GRAFT_REPO_ROOT
for v in dbold dbad; do
  for w in "C5 0.5" "C2 0.15" "C2 0.45" "C2 1.40"; do
    echo "$v $w $(HDB_LIB=ab/libhdb_$v.so python tools/dbscan_c5.py $w 3 2>&1 | tail -1)"
  done
done > gpurun_out/r3z_ab.txt
timeout 1500 python -m pytest tests -m gpu -x -q -k "dbscan or sweep or partition" > gpurun_out/r3z_pytest.txt 2>&1
