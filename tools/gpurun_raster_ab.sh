# GEMM rasterisation A/B at 2048^2: DRAM bytes per launch (ncu launch list of one step, per config)
# and step time (bench.py, interleaved rounds).  Configs: "GROUP:SERP".
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
CFGS=${CFGS:-"8:0 8:1 16:1 32:1"}
for c in $CFGS; do
  G=${c%%:*}; S=${c##*:}
  TSV_GEMM_GROUP=$G TSV_GEMM_SERP=$S timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
    --clock-control none --profile-from-start off --csv --log-file $O/launches_2048_g${G}s${S}.csv \
    python tools/profile_step.py --res 2048 > /dev/null 2>&1; echo "ncu $c exit $?"
  python tools/ncu_summary.py launches $O/launches_2048_g${G}s${S}.csv | head -4
done
for i in 1 2; do
  for c in $CFGS; do
    G=${c%%:*}; S=${c##*:}
    TSV_GEMM_GROUP=$G TSV_GEMM_SERP=$S timeout -s KILL 300 python bench.py --no-cpu-baseline --steps 10 --warmup 3 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$c', d['value'], d['clocks']['sm_mhz'], d['roofline_kernels']['gemm']['achieved'], d['roofline_kernels']['attention']['achieved'], flush=True)"
  done
done
