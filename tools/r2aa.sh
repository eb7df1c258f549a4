cd $GRAFT_REPO_ROOT
VARS="prev2 spf2 sb16 sb16x sb32x" REPS=2 WLS="C3-eps0.07 C3-eps0.12 C3L-eps0.07 C3L-eps0.12" bash tools/ab.sh 2>&1 | tee gpurun_out/r2aa_ab.txt
