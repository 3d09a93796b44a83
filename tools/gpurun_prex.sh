# GEMM epilogue: out0 (fp32 residual) prefetch -- GEMM tests, then whole-step A/B vs the previous .so
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_step.py -m gpu -q -x -p no:cacheprovider > $O/pytest_prex.log 2>&1; echo "pytest exit $?"
tail -3 $O/pytest_prex.log
for cfg in "--model sd3 --res 1024" "--model sd3 --res 2048" "--res 2048"; do
  ARGS="$cfg --steps 10 --warmup 3" ROUNDS=3 bash tools/ab_bench.sh
done
