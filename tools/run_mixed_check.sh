cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests/test_gpu_mixed.py -x -q > gpurun_out/t_mixed.log 2>&1; echo "rc=$?" >> gpurun_out/t_mixed.log
tail -30 gpurun_out/t_mixed.log
timeout -s KILL 300 python bench.py --mix --steps 3 --warmup 2 > gpurun_out/mix.log 2>&1; echo "mix rc=$?"; tail -c 1500 gpurun_out/mix.log
