# secondary bench lines: FLUX 1024^2 / 2048^2 / 4096^2 and SD3 1024^2 / 2048^2 (SP = 1)
cd $GRAFT_REPO_ROOT
O=gpurun_out
for a in "--res 1024" "--res 2048 --steps 10" "--res 4096 --steps 4" "--model sd3 --res 1024" "--model sd3 --res 2048 --steps 10"; do
  timeout -s KILL 600 python bench.py --no-cpu-baseline $a 2>/dev/null | tail -1 >> $O/bench_lines.jsonl; echo "$a exit $?"
done
