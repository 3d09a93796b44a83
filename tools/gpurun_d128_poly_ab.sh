# D=128 poly share, in-step A/B at FLUX 2048^2 (env override of the step's attention impl)
cd $GRAFT_REPO_ROOT
for i in 1 2; do for v in 51 52 50; do
  TSV_ATTN_D128=$v timeout -s KILL 200 python bench.py --no-cpu-baseline --steps 10 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$v', d['value'], d['clocks']['sm_mhz'], d['roofline_kernels']['attention']['achieved'], d['roofline_kernels']['attention']['tensor_util_clock'], flush=True)"
done; done
