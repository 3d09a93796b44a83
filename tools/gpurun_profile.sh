# tests + bench + ncu evidence in one box session
cd $GRAFT_REPO_ROOT
O=gpurun_out
timeout -s KILL 900 python -m pytest tests -m gpu -q -rf --timeout 400 > $O/pytest_gpu.log 2>&1; echo "pytest exit $?"
timeout -s KILL 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke exit $?"
timeout -s KILL 900 python bench.py --steps 10 --warmup 3 > $O/bench.log 2>&1; echo "bench exit $?"
timeout -s KILL 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
   --log-file $O/launches.csv python tools/profile_step.py --res 512 > $O/ncu_launches.log 2>&1; echo "ncu launches exit $?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
   -k regex:gemm_tc -s 5 -c 1 -o $O/prof_gemm_fc1 python tools/profile_step.py --res 512 > $O/ncu_gemm.log 2>&1; echo "ncu gemm exit $?"
timeout -s KILL 600 ncu --set full --clock-control none --profile-from-start off \
   -k regex:attention -s 0 -c 1 -o $O/prof_attn python tools/profile_step.py --res 512 > $O/ncu_attn.log 2>&1; echo "ncu attn exit $?"
timeout -s KILL 600 ncu --set full --clock-control none --profile-from-start off \
   -k regex:"ln_mod|qk_norm" -s 0 -c 2 -o $O/prof_elem python tools/profile_step.py --res 512 > $O/ncu_elem.log 2>&1; echo "ncu elem exit $?"
ls -la $O
