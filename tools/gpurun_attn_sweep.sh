# attention variant sweep: parity tests for the attention kernel + isolated microbench (interleaved rounds)
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k attention > $O/pytest_attn.log 2>&1; echo "pytest exit $?"
tail -3 $O/pytest_attn.log
ATTN_SWEEP=1 ATTN_ROUNDS=${ROUNDS:-3} timeout -s KILL 900 python tools/microbench.py attn > $O/mb_attn.jsonl 2>&1; echo "mb exit $?"
