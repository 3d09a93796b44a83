# split-K evidence: microbench + latency tables (serialised virtual ranks) with and without split-K
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 300 python tools/microbench.py split > $O/mb_split.log 2>&1; cat $O/mb_split.log
for sk in 1 0; do
  TSV_SPLITK=$sk timeout -s KILL 900 python tools/latency_table_model.py --serial --res ${RES:-256,512,1024,2048} --iters 3 \
    --out $O/lt_serial_splitk$sk.json > $O/lt_$sk.log 2>&1; echo "lt splitk=$sk exit $?"
  python -c "import json; d=json.load(open('$O/lt_serial_splitk$sk.json')); print('ms', d['ms']); print('eff', d['efficiency_vs_k1'])"
done
