# whole-step A/B (build/ab/A.so vs B.so), FLUX 2048^2 and SD3 1024^2, interleaved rounds
cd $GRAFT_REPO_ROOT
for cfg in "--res 2048" "--model sd3 --res 1024"; do
  ARGS="$cfg --steps 10 --warmup 3" ROUNDS=${ROUNDS:-3} bash tools/ab_bench.sh
done
