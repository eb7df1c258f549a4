cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:"k_sample_link|k_union" -c 3 -o gpurun_out/r3ff_prof_dbscan python tools/dbscan_c5.py C5 0.5 1 > gpurun_out/r3ff_ncu.log 2>&1
ncu -i gpurun_out/r3ff_prof_dbscan.ncu-rep --page source --csv --print-source cuda,sass -k regex:k_sample_link > gpurun_out/r3ff_cs_sl.csv 2>&1
ncu -i gpurun_out/r3ff_prof_dbscan.ncu-rep --page raw --csv > gpurun_out/r3ff_raw.csv 2>&1
