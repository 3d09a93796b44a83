# GPU test suite + smoke (no bench).  Env: PYTEST_K
cd $GRAFT_REPO_ROOT
O=gpurun_out
timeout -s KILL ${PYTEST_TO:-1500} python -m pytest tests -m gpu -q -rf --timeout 400 ${PYTEST_K:+-k "$PYTEST_K"} > $O/pytest_gpu.log 2>&1; echo "pytest exit $?"
tail -25 $O/pytest_gpu.log
timeout -s KILL 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke exit $?"; tail -2 $O/smoke.log
