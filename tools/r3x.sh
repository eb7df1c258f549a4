cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -x -q -k "dbscan or sweep or partition" > gpurun_out/r3x_pytest.txt 2>&1
python tools/dbscan_c5.py C5 0.5 3 > gpurun_out/r3x_dbscan.txt 2>&1
python tools/dbscan_c5.py C2 0.45 5 >> gpurun_out/r3x_dbscan.txt 2>&1
python tools/dbscan_c5.py C2 1.40 3 >> gpurun_out/r3x_dbscan.txt 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r3x_dbscan_launches.csv python tools/dbscan_c5.py C5 0.5 1 > /dev/null 2>&1
