cd $GRAFT_REPO_ROOT
timeout -s KILL 900 python -m pytest tests -m gpu -q -rf -x --timeout 400 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?"; tail -3 gpurun_out/pytest_gpu.log
GEMM_SHAPES= timeout -s KILL 300 python tools/microbench.py gemm > gpurun_out/mb_gemm.log 2>&1; grep -E '"bn": 0|cublas' gpurun_out/mb_gemm.log
ROUNDS=3 bash tools/ab_bench.sh
