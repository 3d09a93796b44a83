# attention iteration: kernel tests + microbench.  Env: ATTN_IMPLS
cd $GRAFT_REPO_ROOT
O=gpurun_out
timeout -s KILL 150 python -m pytest tests/test_gpu_kernels.py -q -rf -k attention --timeout 200 > $O/pytest_attn.log 2>&1; echo "pytest exit $?"
tail -5 $O/pytest_attn.log
ATTN_IMPLS=${ATTN_IMPLS:-0,12,13,21,22,23,24} timeout -s KILL 200 python tools/microbench.py attn > $O/mb_attn.log 2>&1; echo "mb exit $?"
cat $O/mb_attn.log
