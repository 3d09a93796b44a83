cd $GRAFT_REPO_ROOT
O=gpurun_out
PYARGS="-x -q" bash tools/gpurun_tests.sh
timeout -s KILL 1200 python tools/reshard_bench.py > $O/reshard_bench.jsonl 2> $O/reshard_bench.err; echo "reshard exit $?"
