# SP = 1 tail split (model gain ~1 %, below the default 3 % threshold): whole-step A/B
cd $GRAFT_REPO_ROOT
echo "== FLUX 2048"
ARGS="--steps 10 --warmup 3" ROUNDS=3 ENVS="TSV_KV_GAIN=0.97|TSV_KV_GAIN=0.995" bash tools/ab_envs.sh
echo "== SD3 2048"
ARGS="--model sd3 --res 2048 --steps 10 --warmup 3" ROUNDS=3 ENVS="TSV_KV_GAIN=0.97|TSV_KV_GAIN=0.995" bash tools/ab_envs.sh
