# Table 4 analogue (reshard / step) + the per-rank latency table model (serial virtual ranks)
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 1200 python tools/reshard_bench.py > $O/reshard_bench.jsonl 2> $O/reshard_bench.err; echo "reshard exit $?"
timeout -s KILL 1500 python tools/latency_table_model.py --serial --iters 5 --out $O/latency_table_serial.json > /dev/null 2> $O/ltm.err; echo "ltm exit $?"
