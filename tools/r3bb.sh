cd $GRAFT_REPO_ROOT
WLS="C5-eps0.5" VARS="cur cur:HDB_QLANES=0" REPS=3 bash tools/ab.sh > gpurun_out/r3bb_ab.txt 2>&1
WLS="C3L-eps0.07 C2-eps0.15" VARS="cur cur:HDB_QLANES=0" REPS=1 bash tools/ab.sh >> gpurun_out/r3bb_ab.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/r3bb_pytest.txt 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r3bb_launches_C5.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
