# D=64 attention variants (rotating S): poly share and K/V ring split; guarded small launch first
cd $GRAFT_REPO_ROOT
O=gpurun_out
for I in 96 97; do timeout -s KILL 60 python tools/attn_one.py 4429 24 64 $I > /dev/null 2>&1; echo "one $I $?"; done
timeout -s KILL 400 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k "large_logits or kv_split" > $O/pytest_d64.log 2>&1; echo "pytest $?"; tail -2 $O/pytest_d64.log
ATTN_IMPLS=83,91,92,93,96,97 ATTN_ROUNDS=3 timeout -s KILL 500 python tools/microbench.py attn > $O/mb_d64.jsonl 2>&1; echo "mb $?"
