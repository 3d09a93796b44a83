cd $GRAFT_REPO_ROOT
O=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout -s KILL 1500 python -m pytest tests -m gpu -q -rf --timeout 400 > $O/pytest_gpu.log 2>&1; echo "pytest exit $?"
tail -15 $O/pytest_gpu.log
timeout -s KILL 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke exit $?"; tail -2 $O/smoke.log
timeout -s KILL 600 python bench.py > $O/bench.log 2>&1; echo "bench exit $?"
tail -c 3000 $O/bench.log
