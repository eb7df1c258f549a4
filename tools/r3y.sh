cd $GRAFT_REPO_ROOT
for v in dbold dbnew dbg4 dbsl0 dblab0; do
  for w in "C5 0.5" "C2 0.45" "C2 1.40"; do
    echo "$v $w $(HDB_LIB=ab/libhdb_$v.so python tools/dbscan_c5.py $w 3 2>&1 | tail -1)"
  done
done > gpurun_out/r3y_ab.txt
for v in dbold dbnew; do
  HDB_LIB=ab/libhdb_$v.so ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r3y_launch_${v}_C2.csv python tools/dbscan_c5.py C2 0.45 1 > /dev/null 2>&1
done
