# Same-box A/B of per-rank SP step times (tools/sp_breakdown.py) between build/ab/A.so and B.so,
# interleaved.  Env: ROUNDS, RES, KS, ENV_A, ENV_B
cd $GRAFT_REPO_ROOT
for i in $(seq ${ROUNDS:-3}); do
  for v in A B; do
    if [ $v = A ]; then E="$ENV_A"; else E="$ENV_B"; fi
    env $E TSV_LIB=$PWD/build/ab/$v.so timeout -s KILL 600 python tools/sp_breakdown.py --res ${RES:-512,1024} --ks ${KS:-8} 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print('$v', d['res'], d['k'], d['per_rank_total_ms'], d['per_rank_ms'].get('gemm'), d['per_rank_ms'].get('attention'), flush=True)"
  done
done
