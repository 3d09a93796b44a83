# full GPU suite with the rotating-S D=64 default, then the SD3 1024^2 / 2048^2 step A/B (impl 83 vs 92)
cd $GRAFT_REPO_ROOT
PYARGS="-q -x" TLIM=1500 bash tools/gpurun_tests.sh
for res in 1024 2048; do
for i in 1 2; do
  for v in 83 92; do
    TSV_ATTN_D64=$v timeout -s KILL 200 python bench.py --no-cpu-baseline --model sd3 --res $res --steps 10 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$res', '$v', d['value'], d['clocks']['sm_mhz'], d['roofline_kernels']['attention']['achieved'], d['roofline_kernels']['attention']['tensor_util_clock'], flush=True)"
  done
done
done
