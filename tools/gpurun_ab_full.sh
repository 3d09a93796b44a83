# GPU tests + GEMM microbench (auto tiles) + same-box A/B of bench.py (build/ab/A.so vs B.so)
cd $GRAFT_REPO_ROOT
timeout -s KILL 900 python -m pytest tests -m gpu -q -rf -x --timeout 400 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?"; tail -3 gpurun_out/pytest_gpu.log
timeout -s KILL 300 python tools/microbench.py gemm > gpurun_out/mb_gemm.log 2>&1; grep -E '"bn": 0|cublas' gpurun_out/mb_gemm.log | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print(d['op'][-6:], d['M'], d['N'], d['K'], d['tflops'])"
ROUNDS=${ROUNDS:-3} bash tools/ab_bench.sh
