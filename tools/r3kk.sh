cd $GRAFT_REPO_ROOT
WLS="C2-eps0.45 C3-eps0.07 C3-eps0.20 C2-eps0.15" VARS="cf709029 c4a10139 head" REPS=3 bash tools/ab.sh > gpurun_out/r3kk_ab.txt 2>&1
