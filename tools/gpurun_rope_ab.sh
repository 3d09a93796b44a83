# QK-norm/RoPE epilogue: cos/sin loaded one chunk ahead -- GEMM/step tests + FLUX whole-step A/B
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 1200 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_fused.py tests/test_gpu_step.py -m gpu -q -x -p no:cacheprovider > $O/pytest_rope.log 2>&1; echo "pytest exit $?"
tail -3 $O/pytest_rope.log
for cfg in "--res 2048" "--res 1024"; do
  ARGS="$cfg --steps 10 --warmup 3" ROUNDS=3 bash tools/ab_bench.sh
done
