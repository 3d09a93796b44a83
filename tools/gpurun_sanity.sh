# fresh-checkpoint sanity: probes, GPU tests, smoke, default bench line
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 60 ./tools/probe/mufu_probe > $O/mufu_probe.log 2>&1; cat $O/mufu_probe.log
timeout -s KILL ${PYTEST_TO:-1500} python -m pytest tests -m gpu -q -rf --timeout 400 > $O/pytest_gpu.log 2>&1; echo "pytest exit $?"
tail -8 $O/pytest_gpu.log
timeout -s KILL 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke exit $?"; tail -2 $O/smoke.log
timeout -s KILL 600 python bench.py > $O/bench.log 2>&1; echo "bench exit $?"
tail -c 3000 $O/bench.log
