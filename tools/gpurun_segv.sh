cd $GRAFT_REPO_ROOT
timeout -s KILL 900 python -m pytest tests -m gpu -q -x --timeout 400 2>&1 | tail -3
RES=256,512,1024,2048 bash tools/gpurun_splitk.sh
