cd $GRAFT_REPO_ROOT
O=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi0.txt
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_r2a.log 2>&1; echo "pytest rc $?"
timeout 600 python bench.py --res 2048 --steps 10 --warmup 3 --no-cpu-baseline > $O/bench2048_r2a.log 2>&1; echo "bench rc $?"
ATTN_IMPLS=0 timeout 300 python tools/microbench.py attn > $O/attn_r2a.jsonl 2>&1; echo "attn rc $?"
