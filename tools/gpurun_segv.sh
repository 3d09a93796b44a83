cd $GRAFT_REPO_ROOT
timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -3
timeout -s KILL 300 python tools/microbench.py attnsplit 2>&1 | tee gpurun_out/mb_attnsplit.log
timeout -s KILL 900 python -m pytest tests -m gpu -q -x --timeout 400 2>&1 | tail -3
RES=256,512,1024,2048 bash tools/gpurun_splitk.sh 2>&1 | grep -v gemm_split
