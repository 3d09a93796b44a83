# the driver's bench invocations: reference arm, then ours (N=1 defaults), + the 2-rank bench test
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
( time timeout -s KILL 900 python bench.py --impl reference --gpus 1 --steps ${STEPS:-20} --warmup ${WARM:-5} ) > $O/bench_ref.log 2>&1; echo "ref exit $?"
( time timeout -s KILL 900 python bench.py --gpus 1 --steps ${STEPS:-20} --warmup ${WARM:-5} ) > $O/bench_ours.log 2>&1; echo "ours exit $?"
tail -4 $O/bench_ref.log; tail -4 $O/bench_ours.log
timeout -s KILL 600 python -m pytest tests/test_gpu_ipc.py -m gpu -q -k bench > $O/pytest_bench2.log 2>&1; echo "bench2 exit $?"; tail -3 $O/pytest_bench2.log
