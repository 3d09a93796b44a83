# ncu --set full of the SD3 1024^2 step's GEMMs of one joint block (QKV, proj, fc1, fc2)
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 900 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:gemm -s 3 -c 4 -o $O/prof_sd3_gemm python tools/profile_step.py --res 1024 --model sd3 > $O/ncu_sd3_gemm.log 2>&1; echo "ncu $?"
tail -3 $O/ncu_sd3_gemm.log
