# quick iteration: GPU tests + microbench + bench (no ncu).  Env: PYTEST_K, MB
cd $GRAFT_REPO_ROOT
O=gpurun_out
timeout -s KILL ${PYTEST_TO:-420} python -m pytest tests -m gpu -q -rf -x ${PYTEST_K:+-k "$PYTEST_K"} > $O/pytest_gpu.log 2>&1; echo "pytest exit $?"
tail -15 $O/pytest_gpu.log
timeout -s KILL 300 python tools/microbench.py ${MB:-attn gemm ln qk} > $O/microbench.log 2>&1; echo "microbench exit $?"
cat $O/microbench.log
timeout -s KILL 400 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/bench.log 2>&1; echo "bench exit $?"
tail -c 2500 $O/bench.log
