cd $GRAFT_REPO_ROOT
VARS="v3 cs csel el" REPS=3 WLS="C5-eps0.5 C2-eps0.45 C2-eps1.40" bash tools/ab.sh 2>&1 | tee gpurun_out/r2g_ab.txt
