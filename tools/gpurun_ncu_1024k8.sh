# ncu at FLUX 1024^2 k = 8 (SURVEY §8(d) counters): launch list + attention / GEMM full captures
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  --profile-from-start off --csv --log-file $O/launches_1024_k8.csv python tools/profile_step.py --res 1024 --k 8 > $O/ncu_l1024k8.log 2>&1; echo "launches exit $?"
python tools/ncu_summary.py launches $O/launches_1024_k8.csv > $O/launches_1024_k8_summary.txt 2>&1
timeout -s KILL 600 ncu --set full --clock-control none --profile-from-start off -k regex:attention -s 0 -c 1 \
  -o $O/prof_attn_1024_k8 python tools/profile_step.py --res 1024 --k 8 > $O/ncu_a1024k8.log 2>&1; echo "attn exit $?"
timeout -s KILL 600 ncu --set full --clock-control none --profile-from-start off -k regex:gemm_tc -s 10 -c 4 \
  -o $O/prof_gemm_1024_k8 python tools/profile_step.py --res 1024 --k 8 > $O/ncu_g1024k8.log 2>&1; echo "gemm exit $?"
python tools/ncu_summary.py report $O/prof_attn_1024_k8.ncu-rep $O/prof_gemm_1024_k8.ncu-rep > $O/ncu_full_summary_1024_k8.txt 2>&1
mkdir -p /tmp/r && mv $O/*.ncu-rep /tmp/r/
