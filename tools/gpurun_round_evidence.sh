# Round evidence in one call: default bench line, secondary bench lines, per-rank SP breakdown and
# serialised latency tables (FLUX, SD3).  ncu: tools/gpurun_round_ncu.sh (separate call)
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
rm -f $O/bench_lines.jsonl
timeout -s KILL 600 python bench.py > $O/bench_default.log 2>&1; echo "bench exit $?"; tail -1 $O/bench_default.log | cut -c1-300
bash tools/gpurun_bench_lines.sh
timeout -s KILL 900 python tools/sp_breakdown.py --out $O/sp_breakdown.jsonl > /dev/null 2>&1; echo "sp flux exit $?"
timeout -s KILL 900 python tools/sp_breakdown.py --model sd3 --res 1024,2048 --out $O/sp_breakdown_sd3.jsonl > /dev/null 2>&1; echo "sp sd3 exit $?"
timeout -s KILL 1200 python tools/latency_table_model.py --serial --res 256,512,1024,2048,4096 --iters 3 --out $O/latency_table_serial.json > $O/lt.log 2>&1; echo "lt flux exit $?"
timeout -s KILL 900 python tools/latency_table_model.py --model sd3 --serial --res 256,512,1024,2048,4096 --iters 3 --out $O/latency_table_serial_sd3.json > $O/lt_sd3.log 2>&1; echo "lt sd3 exit $?"
