# minimax quadratic vs cubic polynomial exp2 (saturating-FFMA form): parity, isolated, in-step
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k "attention" -p no:cacheprovider > $O/pytest_quad.log 2>&1; echo "pytest exit $?"
tail -2 $O/pytest_quad.log
echo "== SD3 2048"
ARGS="--model sd3 --res 2048 --steps 10 --warmup 3" ROUNDS=3 ENVS="TSV_ATTN_D64=96|TSV_ATTN_D64=103|TSV_ATTN_D64=104" bash tools/ab_envs.sh
echo "== FLUX 2048"
ARGS="--steps 10 --warmup 3" ROUNDS=3 ENVS="TSV_ATTN_D128=56|TSV_ATTN_D128=64" bash tools/ab_envs.sh
