# quick iteration: kernel tests + step tests + microbench + bench (no ncu)
cd $GRAFT_REPO_ROOT
O=gpurun_out
timeout -s KILL 900 python -m pytest tests -m gpu -q -rf --timeout 400 -x ${PYTEST_K:+-k "$PYTEST_K"} > $O/pytest_gpu.log 2>&1; echo "pytest exit $?"
tail -15 $O/pytest_gpu.log
timeout -s KILL 600 python tools/microbench.py ${MB:-attn gemm ln qk} > $O/microbench.log 2>&1; echo "microbench exit $?"
cat $O/microbench.log | tail -40
timeout -s KILL 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/bench.log 2>&1; echo "bench exit $?"
tail -c 1500 $O/bench.log
