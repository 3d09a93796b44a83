# ncu evidence: per-launch list of one step at RES (time + DRAM bytes) + full captures of the top kernels
cd $GRAFT_REPO_ROOT
O=gpurun_out
RES=${RES:-512}
MODEL=${MODEL:-flux}
TAG=${MODEL/flux/}${RES}
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
   --profile-from-start off --csv --log-file $O/launches_$TAG.csv python tools/profile_step.py --res $RES --model $MODEL > $O/ncu_launches_$TAG.log 2>&1; echo "launches exit $?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:gemm_tc -s ${GS:-6} -c 2 -o $O/prof_gemm_$TAG python tools/profile_step.py --res $RES --model $MODEL > $O/ncu_gemm_$TAG.log 2>&1; echo "gemm exit $?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:attention -s 0 -c 1 -o $O/prof_attn_$TAG python tools/profile_step.py --res $RES --model $MODEL > $O/ncu_attn_$TAG.log 2>&1; echo "attn exit $?"
timeout -s KILL 600 ncu --set full --clock-control none --profile-from-start off \
   -k regex:ln_mod -s 0 -c 1 -o $O/prof_ln_$TAG python tools/profile_step.py --res $RES --model $MODEL > $O/ncu_ln_$TAG.log 2>&1; echo "ln exit $?"
ls -la $O
