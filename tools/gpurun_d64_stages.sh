# D=64 rotating-S attention: 4 vs 6 joint K/V stages (guarded launch, parity, microbench, SD3 step A/B)
cd $GRAFT_REPO_ROOT
O=gpurun_out
for I in 96 97; do timeout -s KILL 60 python tools/attn_one.py 4429 24 64 $I > /dev/null 2>&1; echo "one $I $?"; done
timeout -s KILL 60 python tools/attn_one.py 4429 24 64 96 > /dev/null 2>&1 || exit 1
ATTN_IMPLS=92,93,96,97 ATTN_ROUNDS=3 timeout -s KILL 400 python tools/microbench.py attn > $O/mb_d64_st.jsonl 2>&1; echo "mb $?"
for i in 1 2; do for v in 92 96; do
  TSV_ATTN_D64=$v timeout -s KILL 200 python bench.py --no-cpu-baseline --model sd3 --res 2048 --steps 10 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$v', d['value'], d['clocks']['sm_mhz'], d['roofline_kernels']['attention']['tensor_util_clock'], flush=True)"
done; done
