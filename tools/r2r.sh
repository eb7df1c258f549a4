cd $GRAFT_REPO_ROOT
VARS="base2 ps3" REPS=3 WLS="C5-eps0.5 C2-eps0.45" bash tools/ab.sh 2>&1 | tee gpurun_out/r2r_ab.txt
