cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/r2k_pytest.txt 2>&1
echo "PYTEST: $(tail -1 gpurun_out/r2k_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/r2k_pytest.txt | head -8
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --workload C5-eps0.5 --steps 3 --warmup 1 --e2e-steps 1 --no-cpu-baseline > gpurun_out/r2k_torchrun2.json 2> gpurun_out/r2k_torchrun2.err
echo "TORCHRUN rc=$?"; tail -c 1500 gpurun_out/r2k_torchrun2.json; tail -5 gpurun_out/r2k_torchrun2.err
