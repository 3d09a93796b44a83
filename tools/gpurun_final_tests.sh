# full GPU suite (incl. the 2048^2 golden), then an SD3 step A/B of the D=64 attention (env override)
cd $GRAFT_REPO_ROOT
O=gpurun_out
PYARGS="-q -rs" TLIM=1800 bash tools/gpurun_tests.sh
for i in 1 2 3; do
  for v in 83 92; do
    TSV_ATTN_D64=$v timeout -s KILL 300 python bench.py --no-cpu-baseline --model sd3 --res ${RES:-1024} --steps 10 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$v', d['value'], d['clocks']['sm_mhz'], d['roofline_kernels']['attention']['achieved'], d['time_share'], flush=True)"
  done
done
