# ncu --set full of the FLUX 2048^2 step's GEMMs of one double block (QKV, proj, fc1, fc2) and one single block (linear1, linear2)
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 1200 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:gemm -s 1 -c 4 -o $O/prof_flux_gemm python tools/profile_step.py --res 2048 > $O/ncu_flux_gemm.log 2>&1; echo "ncu $?"
timeout -s KILL 1200 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:gemm -s 77 -c 2 -o $O/prof_flux_gemm_single python tools/profile_step.py --res 2048 > $O/ncu_flux_gemm2.log 2>&1; echo "ncu single $?"
