# attention KV tail split: parity tests, then per-rank breakdown at SP = 2 / 4 / 8 (FLUX, SD3 2048^2)
# with TSV_KV_TAIL=0 (uniform splits, round 2's plan) vs 1, interleaved
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 900 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k "attention" -p no:cacheprovider > $O/pytest_tail.log 2>&1; echo "pytest exit $?"
tail -3 $O/pytest_tail.log
for i in 1 2; do
  for v in 0 1; do
    TSV_KV_TAIL=$v TSV_VIRTUAL_SERIAL=1 timeout -s KILL 900 python tools/sp_breakdown.py --res 2048 --ks 2,4,8 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print('tail=$v', d['model'], d['res'], d['k'], d['per_rank_total_ms'], d['per_rank_ms']['attention'], d['tflops']['attention'], flush=True)"
    TSV_KV_TAIL=$v TSV_VIRTUAL_SERIAL=1 timeout -s KILL 900 python tools/sp_breakdown.py --model sd3 --res 2048 --ks 2,4,8 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print('tail=$v', d['model'], d['res'], d['k'], d['per_rank_total_ms'], d['per_rank_ms']['attention'], d['tflops']['attention'], flush=True)"
  done
done
