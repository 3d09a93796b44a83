# A/B/C... of whole steps under several environments (same .so), interleaved rounds.
# Env: ROUNDS, ARGS, ENVS ("|"-separated, e.g. ENVS="TSV_ATTN_D128=51|TSV_ATTN_D128=56")
cd $GRAFT_REPO_ROOT
IFS='|' read -ra EL <<< "$ENVS"
for i in $(seq ${ROUNDS:-3}); do
  for E in "${EL[@]}"; do
    env $E timeout -s KILL 300 python bench.py --no-cpu-baseline ${ARGS:---steps 20} 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); rk=d['roofline_kernels']; print('$E |', d['value'], d['clocks']['sm_mhz'], rk['gemm']['achieved'], rk['attention']['achieved'], d['time_share']['attention'], flush=True)"
  done
done
