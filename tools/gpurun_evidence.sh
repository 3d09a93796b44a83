# Refresh the ncu evidence: launch lists + full captures at FLUX 512^2, FLUX 2048^2, SD3 1024^2
cd $GRAFT_REPO_ROOT
RES=512 bash tools/gpurun_ncu.sh
RES=2048 GS=6 bash tools/gpurun_ncu.sh
MODEL=sd3 RES=1024 bash tools/gpurun_ncu.sh
ls -la gpurun_out
