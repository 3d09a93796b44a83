# per-rank kernel efficiency at SP = 8 (FLUX 2048^2, 8 virtual ranks serialised): ncu launch list with
# grid sizes + per-class breakdown at k = 1 / 8
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,launch__grid_size,dram__bytes_read.sum,dram__bytes_write.sum \
  --clock-control none --profile-from-start off --csv --log-file $O/launches_2048_k8.csv \
  python tools/profile_step.py --res 2048 --k 8 > /dev/null 2>&1; echo "ncu k8 $?"
TSV_VIRTUAL_SERIAL=1 timeout -s KILL 900 python tools/sp_breakdown.py --res 2048 --ks 1,8 --out $O/sp_breakdown_2048.jsonl > /dev/null 2> $O/spb.err; echo "spb $?"
cat $O/sp_breakdown_2048.jsonl
