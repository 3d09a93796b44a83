# ncu evidence for the SP = 8 per-rank kernels (k virtual ranks; ncu serialises the launches):
# launch lists at FLUX 2048^2 and 512^2 (k = 8), full captures of the KV-split attention and a
# split-K GEMM, summarised on the box
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
for r in 2048 512; do
  timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --profile-from-start off --csv --log-file $O/launches_${r}_k8.csv python tools/profile_step.py --res $r --k 8 > $O/ncu_launches_${r}_k8.log 2>&1; echo "launches $r exit $?"
  python tools/ncu_summary.py launches $O/launches_${r}_k8.csv > $O/launches_${r}_k8_summary.txt 2>&1
done
timeout -s KILL 600 ncu --set full --clock-control none --profile-from-start off -k regex:attention -s 0 -c 1 \
  -o $O/prof_attn_2048_k8 python tools/profile_step.py --res 2048 --k 8 > $O/ncu_attn_k8.log 2>&1; echo "attn exit $?"
timeout -s KILL 600 ncu --set full --clock-control none --profile-from-start off -k regex:gemm_tc -s 2 -c 6 \
  -o $O/prof_gemm_512_k8 python tools/profile_step.py --res 512 --k 8 > $O/ncu_gemm_k8.log 2>&1; echo "gemm exit $?"
python tools/ncu_summary.py report $O/prof_attn_2048_k8.ncu-rep $O/prof_gemm_512_k8.ncu-rep > $O/ncu_full_summary_k8.txt 2>&1
mkdir -p /tmp/ncu_reps && mv $O/*.ncu-rep /tmp/ncu_reps/
du -sh $O
