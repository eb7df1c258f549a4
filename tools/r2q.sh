cd $GRAFT_REPO_ROOT
s=$(date +%s); timeout 900 python bench.py > gpurun_out/r2q_bench_default.json 2> gpurun_out/r2q_bench_default.err; echo "default bench rc=$? $(( $(date +%s) - s )) s"
s=$(date +%s); timeout 900 python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/r2q_ref.json 2> gpurun_out/r2q_ref.err; echo "reference rc=$? $(( $(date +%s) - s )) s"
timeout 1800 python tools/traffic.py > gpurun_out/r2q_traffic.log 2>&1; echo "traffic rc=$?"; tail -3 gpurun_out/r2q_traffic.log
