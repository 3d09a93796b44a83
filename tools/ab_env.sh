# A/B of whole steps under two environments (same .so): alternate bench.py runs with ENV_A / ENV_B.
# Env: ROUNDS, ARGS, ENV_A, ENV_B (e.g. ENV_A="TSV_ATTN_D128=51" ENV_B="TSV_ATTN_D128=52")
cd $GRAFT_REPO_ROOT
for i in $(seq ${ROUNDS:-3}); do
  for v in A B; do
    if [ $v = A ]; then E="$ENV_A"; else E="$ENV_B"; fi
    env $E timeout -s KILL 300 python bench.py --no-cpu-baseline ${ARGS:---steps 20} 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$v', '$E', d['value'], d['clocks']['sm_mhz'], d.get('attention_tflops'), d['time_share']['attention'], flush=True)"
  done
done
