# attention variant A/B: parity tests for the attention kernels + isolated microbench of ATTN_IMPLS
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -rf -k attention > $O/pytest_attn.log 2>&1; echo "pytest exit $?"
tail -5 $O/pytest_attn.log
ATTN_IMPLS=${ATTN_IMPLS:-0,50,51,52,53} timeout -s KILL 600 python tools/microbench.py attn > $O/mb_attn.log 2>&1; echo "mb exit $?"
cat $O/mb_attn.log
