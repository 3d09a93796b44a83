# round-2 final evidence: GPU suite, parity vs all goldens, bench lines, ncu launch lists + top-kernel
# captures, per-rank latency tables (FLUX, SD3), reshard table
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
PYARGS="-q -rs" TLIM=1800 bash tools/gpurun_tests.sh
timeout -s KILL 900 python tools/parity_report.py > $O/parity.jsonl 2> $O/parity.err; echo "parity $?"
timeout -s KILL 600 python bench.py > $O/bench_2048.json 2> $O/bench_2048.err; echo "bench 2048 $?"
: > $O/bench_lines.jsonl
for a in "--res 512" "--res 1024" "--model sd3 --res 1024" "--model sd3 --res 2048" "--res 4096 --steps 5"; do
  timeout -s KILL 600 python bench.py --no-cpu-baseline --steps 10 $a >> $O/bench_lines.jsonl 2>> $O/bench_lines.err; echo "bench $a $?"
done
for r in 2048 512; do
  timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
     --profile-from-start off --csv --log-file $O/launches_$r.csv python tools/profile_step.py --res $r > /dev/null 2>&1; echo "launches $r $?"
done
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
   --profile-from-start off --csv --log-file $O/launches_sd31024.csv python tools/profile_step.py --res 1024 --model sd3 > /dev/null 2>&1; echo "launches sd3 $?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:attention -s 0 -c 1 -o $O/prof_attn_2048 python tools/profile_step.py --res 2048 > /dev/null 2>&1; echo "attn full $?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:attention -s 0 -c 1 -o $O/prof_attn_sd32048 python tools/profile_step.py --res 2048 --model sd3 > /dev/null 2>&1; echo "attn sd3 full $?"
timeout -s KILL 1200 python tools/latency_table_model.py --serial --iters 5 --out $O/latency_table_serial.json > /dev/null 2> $O/ltm.err; echo "ltm $?"
timeout -s KILL 1200 python tools/latency_table_model.py --serial --model sd3 --iters 5 --out $O/latency_table_serial_sd3.json > /dev/null 2> $O/ltm_sd3.err; echo "ltm sd3 $?"
timeout -s KILL 900 python tools/reshard_bench.py > $O/reshard_bench.jsonl 2> $O/reshard_bench.err; echo "reshard $?"
