# GEMM QKV epilogue A/B (A.so before, B.so after): fused-epilogue parity tests on B, qkv microbench, step A/B
cd $GRAFT_REPO_ROOT
TSV_LIB=$PWD/build/ab/B.so timeout -s KILL 400 python -m pytest tests/test_gpu_fused.py tests/test_gpu_kernels.py -m gpu -q -x -k "qk or fused or epilogue" 2>&1 | tail -2
for v in A B A B; do echo $v; TSV_LIB=$PWD/build/ab/$v.so timeout -s KILL 200 python tools/microbench.py qkv; done
ARGS="--steps 10" ROUNDS=3 bash tools/ab_bench.sh
