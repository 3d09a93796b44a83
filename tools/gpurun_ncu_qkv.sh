# ncu --set full + source of the FLUX 2048^2 QKV GEMM (double block 0, fused QK-norm/RoPE epilogue) and fc1
cd $GRAFT_REPO_ROOT
O=gpurun_out
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:gemm_tc -s 1 -c 1 -o $O/prof_qkv_2048 python tools/profile_step.py --res 2048 > /dev/null 2>&1; echo "qkv $?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:gemm_tc -s 3 -c 1 -o $O/prof_fc1_2048 python tools/profile_step.py --res 2048 > /dev/null 2>&1; echo "fc1 $?"
