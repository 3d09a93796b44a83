cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "split" 2>&1 | tail -2
timeout 900 python -m pytest tests -m gpu -q -x --timeout 400 2>&1 | tail -2
for sk in 1 0; do TSV_SPLITK=$sk timeout 600 python tools/sp_breakdown.py --res 256,512,1024 --ks 1,4,8 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print('splitk=$sk', d['res'], d['k'], d['per_rank_total_ms'], d['per_rank_ms'].get('gemm'))"; done
