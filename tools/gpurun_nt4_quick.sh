# quick guarded check of the four-tile D=64 attention: one small launch per impl under a 60 s timeout,
# then the parity tests and the microbench only if that worked
cd $GRAFT_REPO_ROOT
O=gpurun_out
for I in 93 99; do
  timeout -s KILL 60 python tools/attn_one.py 1357 4 64 $I > $O/nt4_one_$I.log 2>&1; echo "one $I exit $?"
done
timeout -s KILL 60 python tools/attn_one.py 1357 4 64 93 > /dev/null 2>&1 || exit 1
timeout -s KILL 300 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k "attention" > $O/pytest_attn_nt4.log 2>&1; echo "pytest exit $?"; tail -3 $O/pytest_attn_nt4.log
TSV_LIB=$PWD/build/ab/A.so ATTN_IMPLS=83 ATTN_ROUNDS=2 timeout -s KILL 300 python tools/microbench.py attn > $O/mb_nt4_A.jsonl 2>&1
ATTN_IMPLS=83,92,93,94,99 ATTN_ROUNDS=2 timeout -s KILL 300 python tools/microbench.py attn > $O/mb_nt4_B.jsonl 2>&1; echo "mb exit $?"
