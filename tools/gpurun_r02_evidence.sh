# round-2 evidence: bench lines (2048^2 default, 512^2, SD3 1024^2/2048^2), ncu launch lists of one step
# (2048^2, 512^2, SD3 1024^2) and ncu --set full of the top kernels at 2048^2
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 600 python bench.py --no-cpu-baseline > $O/bench_2048.json 2> $O/bench_2048.err; echo "bench 2048 $?"
for a in "--res 512" "--model sd3 --res 1024" "--model sd3 --res 2048" "--res 1024" "--res 4096 --steps 5"; do
  timeout -s KILL 600 python bench.py --no-cpu-baseline --steps 10 $a >> $O/bench_lines.jsonl 2>> $O/bench_lines.err; echo "bench $a $?"
done
for r in 2048 512; do
  RES=$r timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
     --profile-from-start off --csv --log-file $O/launches_$r.csv python tools/profile_step.py --res $r > /dev/null 2>&1; echo "launches $r $?"
done
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
   --profile-from-start off --csv --log-file $O/launches_sd31024.csv python tools/profile_step.py --res 1024 --model sd3 > /dev/null 2>&1; echo "launches sd3 $?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:gemm_tc -s 6 -c 2 -o $O/prof_gemm_2048 python tools/profile_step.py --res 2048 > /dev/null 2>&1; echo "gemm full $?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:attention -s 0 -c 1 -o $O/prof_attn_2048 python tools/profile_step.py --res 2048 > /dev/null 2>&1; echo "attn full $?"
timeout -s KILL 600 ncu --set full --clock-control none --profile-from-start off \
   -k regex:ln_mod -s 0 -c 1 -o $O/prof_ln_2048 python tools/profile_step.py --res 2048 > /dev/null 2>&1; echo "ln full $?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:attention -s 0 -c 1 -o $O/prof_attn_sd31024 python tools/profile_step.py --res 1024 --model sd3 > /dev/null 2>&1; echo "attn sd3 full $?"
