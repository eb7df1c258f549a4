cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,memory.total --format=csv > gpurun_out/r2a_gpu.txt; nproc >> gpurun_out/r2a_gpu.txt; free -g >> gpurun_out/r2a_gpu.txt
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 --durations=40 > gpurun_out/r2a_pytest.txt 2>&1
echo "PYTEST rc=$?: $(tail -1 gpurun_out/r2a_pytest.txt)"
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r2a_bench.json 2> gpurun_out/r2a_bench.err
echo "BENCH rc=$?"; tail -c 600 gpurun_out/r2a_bench.json
