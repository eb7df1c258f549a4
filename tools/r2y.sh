cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/r2y_pytest.txt 2>&1
echo "PYTEST: $(tail -1 gpurun_out/r2y_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/r2y_pytest.txt | head -8
VARS="prev2 spf" REPS=3 WLS="C3-eps0.07 C3-eps0.12 C3L-eps0.07 C3L-eps0.12 C5-eps0.5" bash tools/ab.sh 2>&1 | tee gpurun_out/r2y_ab.txt
