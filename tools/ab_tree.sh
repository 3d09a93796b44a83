# Same-box A/B of two source trees: A = build/ab/old (an older checkout with its own libtsv.so), B = this tree.
# Env: ROUNDS, ARGS, ENV_B (environment for B's runs, e.g. "TSV_SPLITK=0 TSV_ATTN_D128=52")
cd $GRAFT_REPO_ROOT
for i in $(seq ${ROUNDS:-3}); do
  for v in A B; do
    if [ $v = A ]; then d=build/ab/old; else d=.; fi
    if [ $v = A ]; then E=; else E="$ENV_B"; fi
    (cd $d && env $E timeout -s KILL 300 python bench.py --no-cpu-baseline ${ARGS:---steps 20} 2>/dev/null) | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$v', d['value'], d['clocks']['sm_mhz'], d['roofline']['achieved'], d.get('attention_tflops'), d['time_share'], flush=True)"
  done
done
