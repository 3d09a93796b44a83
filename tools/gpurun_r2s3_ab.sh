# Whole-step A/B of attention variants (saturating-FFMA polynomial exp2 vs round 2's defaults):
# attention parity tests, then FLUX 2048^2 (D = 128) and SD3 2048^2 (D = 64) interleaved rounds.
# (The first run of this script also A/B'd GEMM L2 eviction-priority hints -- TSV_L2_KEEP_MB, since
# removed: profiles/r02/ab_psat_l2hint.txt, ab_l2last_d128psat.txt.)
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 900 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k attention -p no:cacheprovider > $O/pytest_psat.log 2>&1; echo "pytest exit $?"
tail -2 $O/pytest_psat.log
echo "== FLUX 2048"
ARGS="--steps 10 --warmup 3" ROUNDS=3 ENVS="TSV_ATTN_D128=51|TSV_ATTN_D128=55|TSV_ATTN_D128=56" bash tools/ab_envs.sh
echo "== SD3 2048"
ARGS="--model sd3 --res 2048 --steps 10 --warmup 3" ROUNDS=3 ENVS="TSV_ATTN_D64=92|TSV_ATTN_D64=96|TSV_ATTN_D64=95" bash tools/ab_envs.sh
