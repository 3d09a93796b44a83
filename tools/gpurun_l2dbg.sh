cd $GRAFT_REPO_ROOT
python - <<'PY'
import ctypes
rt = ctypes.CDLL('libcudart.so.12')
v = ctypes.c_int()
rt.cudaDeviceGetAttribute(ctypes.byref(v), 109, 0)   # cudaDevAttrMaxAccessPolicyWindowSize
print('max window', v.value)
PY
TSV_GEMM_L2PERSIST=1 timeout -s KILL 120 python bench.py --no-cpu-baseline --steps 3 --res 512 2>&1 | tail -3
