# D = 128: 2 vs 3 vs 4 of 8 exp2 pairs by the saturating-FFMA cubic (impl 56 / 57 / 58): isolated + in-step
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k "test_attention and not split and not tail" -p no:cacheprovider > $O/pytest_p3.log 2>&1; echo "pytest exit $?"
tail -2 $O/pytest_p3.log
ATTN_IMPLS=56,57,58 ATTN_ROUNDS=3 timeout -s KILL 600 python tools/microbench.py attn 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    if d['D']==128: print(d['L'],d['H'],d['impl'],d['ms'],d['tflops'])"
echo "== FLUX 2048"
ARGS="--steps 10 --warmup 3" ROUNDS=3 ENVS="TSV_ATTN_D128=56|TSV_ATTN_D128=57|TSV_ATTN_D128=58" bash tools/ab_envs.sh
