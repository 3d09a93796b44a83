# D = 128 MMA issue order alternating the query tile served first (impl 57) vs 56
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k "attention" -p no:cacheprovider > $O/pytest_alt.log 2>&1; echo "pytest exit $?"
tail -2 $O/pytest_alt.log
ATTN_IMPLS=56,57 ATTN_ROUNDS=3 timeout -s KILL 600 python tools/microbench.py attn 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    if d['D']==128: print(d['L'],d['H'],d['impl'],d['ms'],d['tflops'])"
echo "== FLUX 2048"
ARGS="--steps 10 --warmup 3" ROUNDS=3 ENVS="TSV_ATTN_D128=56|TSV_ATTN_D128=57" bash tools/ab_envs.sh
