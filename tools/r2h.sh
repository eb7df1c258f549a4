cd $GRAFT_REPO_ROOT
VARS="csel csel:HDB_FUSED_CHUNK=16 csel:HDB_FUSED_CHUNK=8 csel:HDB_FUSED_CHUNK=4 csel:HDB_FUSED_CHUNK=64" REPS=2 WLS="C5-eps0.5 C2-eps0.45" bash tools/ab.sh 2>&1 | tee gpurun_out/r2h_ab.txt
