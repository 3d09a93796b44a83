set -x
cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -q -rf --timeout 200 > gpurun_out/pytest_kernels.log 2>&1
echo "kernels exit $?"
timeout -s KILL 600 python -m pytest tests/test_gpu_step.py -q -rf -s --timeout 300 > gpurun_out/pytest_step.log 2>&1
echo "step exit $?"
timeout -s KILL 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
echo "smoke exit $?"
timeout -s KILL 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench.log 2>&1
echo "bench exit $?"
tail -3 gpurun_out/pytest_kernels.log gpurun_out/pytest_step.log gpurun_out/smoke.log gpurun_out/bench.log
