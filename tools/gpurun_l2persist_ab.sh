# GEMM L2-persisting weight windows: DRAM bytes (ncu launch list) and step time, off / max carve-out / 32 MB
cd $GRAFT_REPO_ROOT
O=gpurun_out
python -c "
import torch; p=torch.cuda.get_device_properties(0); print('L2', p.L2_cache_size)" 2>/dev/null
python - <<'PY'
import ctypes
rt = ctypes.CDLL('libcudart.so.12')
v = ctypes.c_int()
rt.cudaDeviceGetAttribute(ctypes.byref(v), 108, 0)   # cudaDevAttrMaxPersistingL2CacheSize
print('max persisting L2', v.value)
PY
for cfg in "0:0" "1:0" "1:32"; do
  P=${cfg%%:*}; MB=${cfg##*:}
  if [ $MB = 0 ]; then unset TSV_L2_PERSIST_MB; else export TSV_L2_PERSIST_MB=$MB; fi
  TSV_GEMM_L2PERSIST=$P timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
    --clock-control none --profile-from-start off --csv --log-file $O/launches_2048_l2_${P}_${MB}.csv \
    python tools/profile_step.py --res 2048 > /dev/null 2>&1; echo "ncu $cfg $?"
  python tools/ncu_summary.py launches $O/launches_2048_l2_${P}_${MB}.csv 2>/dev/null | head -4
done
unset TSV_L2_PERSIST_MB
for i in 1 2; do
  for cfg in "0:0" "1:0" "1:32"; do
    P=${cfg%%:*}; MB=${cfg##*:}
    if [ $MB = 0 ]; then unset TSV_L2_PERSIST_MB; else export TSV_L2_PERSIST_MB=$MB; fi
    TSV_GEMM_L2PERSIST=$P timeout -s KILL 300 python bench.py --no-cpu-baseline --steps 10 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); rk=d['roofline_kernels']; print('$cfg', d['value'], d['clocks']['sm_mhz'], rk['gemm']['achieved'], rk['attention']['achieved'], flush=True)"
  done
done
