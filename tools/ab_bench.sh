# A/B: alternate bench.py runs between build/ab/A.so and build/ab/B.so.  Env: ROUNDS, ARGS
cd $GRAFT_REPO_ROOT
for i in $(seq ${ROUNDS:-3}); do
  for v in A B; do
    TSV_LIB=$PWD/build/ab/$v.so timeout -s KILL 300 python bench.py --no-cpu-baseline ${ARGS:---steps 20} 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$v', d['value'], d['clocks']['sm_mhz'], d['time_share'])"
  done
done
