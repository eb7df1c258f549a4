cd $GRAFT_REPO_ROOT
VARS="csel w4 w4b9 w4b10" REPS=2 WLS="C5-eps0.5 C2-eps0.45 C2-eps1.40 C2-eps0.15" bash tools/ab.sh 2>&1 | tee gpurun_out/r2i_ab.txt
