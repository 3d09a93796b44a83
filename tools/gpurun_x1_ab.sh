# GEMM epilogue out0 rows prefetched one chunk ahead (no pre-wait load): tests + whole-step A/B
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 1200 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_step.py tests/test_gpu_sd3.py -m gpu -q -x -p no:cacheprovider > $O/pytest_x1.log 2>&1; echo "pytest exit $?"
tail -3 $O/pytest_x1.log
for cfg in "--model sd3 --res 1024" "--model sd3 --res 2048" "--res 2048"; do
  ARGS="$cfg --steps 10 --warmup 3" ROUNDS=3 bash tools/ab_bench.sh
done
