# the GPU test suite (+ smoke), logs under gpurun_out/
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL ${TLIM:-1500} python -m pytest tests -m gpu -q ${PYARGS:--x} > $O/pytest_gpu.log 2>&1; echo "pytest exit $?"
tail -15 $O/pytest_gpu.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke exit $?"; tail -2 $O/smoke.log
