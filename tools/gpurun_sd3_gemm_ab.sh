# SD3 1024^2 step: the GEMM planner's tile choice vs forced tile widths / CTA pairing (env A/B)
cd $GRAFT_REPO_ROOT
for i in 1 2; do
  for cfg in "0:-1" "128:1" "256:0" "256:1" "128:0"; do
    BN=${cfg%%:*}; PR=${cfg##*:}
    TSV_GEMM_BN=$BN TSV_GEMM_PAIR=$PR timeout -s KILL 200 python bench.py --no-cpu-baseline --model sd3 --res 1024 --steps 10 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$cfg', d['value'], d['clocks']['sm_mhz'], d['roofline_kernels']['gemm']['achieved'], d['roofline_kernels']['gemm']['tensor_util_clock'], flush=True)"
  done
done
