cd $GRAFT_REPO_ROOT
O=gpurun_out
TSV_ATTN_D64=92 timeout -s KILL 120 python bench.py --no-cpu-baseline --model sd3 --res 1024 --steps 3 > $O/rs_bench.log 2>&1; echo "bench rc $?"; tail -5 $O/rs_bench.log
timeout -s KILL 300 python -m pytest tests/test_gpu_sd3.py -m gpu -q -x > $O/rs_sd3.log 2>&1; echo "sd3 tests rc $?"; tail -5 $O/rs_sd3.log
