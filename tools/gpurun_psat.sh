# saturating-FFMA poly exp2 variants: attention parity tests + interleaved isolated microbench
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 900 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k attention -p no:cacheprovider > $O/pytest_psat.log 2>&1; echo "pytest exit $?"
tail -3 $O/pytest_psat.log
ATTN_IMPLS=${IMPLS:-92,93,95,96,97,51,55,56} ATTN_ROUNDS=${ROUNDS:-3} timeout -s KILL 900 python tools/microbench.py attn > $O/mb_psat.jsonl 2>&1; echo "mb exit $?"
cat $O/mb_psat.jsonl | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: print(l.strip()); continue
    print(d['L'],d['H'],d['D'],d['impl'],d['ms'],d['tflops'])"
