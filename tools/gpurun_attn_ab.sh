# attention A/B: build/ab/A.so (before) vs build/ab/B.so (after): parity tests on B, then isolated
# microbench of IMPLS_A on A and IMPLS_B on B, ROUNDS alternations
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
TSV_LIB=$PWD/build/ab/B.so timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -k attention > $O/pytest_attn_ab.log 2>&1; echo "pytest exit $?"; tail -2 $O/pytest_attn_ab.log
: > $O/mb_attn_ab.jsonl
for i in $(seq ${ROUNDS:-2}); do
  for v in A B; do
    if [ $v = A ]; then IM=${IMPLS_A:-0}; else IM=${IMPLS_B:-0}; fi
    TSV_LIB=$PWD/build/ab/$v.so ATTN_IMPLS=$IM ATTN_ROUNDS=1 timeout -s KILL 600 python tools/microbench.py attn 2>&1 | sed "s/^{/{\"lib\": \"$v\", /" >> $O/mb_attn_ab.jsonl
  done
done
echo done
