# attention diagnostics: the kernel with no exponential (impl 59) / all-polynomial exp2 (58) vs the
# step's default, isolated microbench + ncu tensor-pipe / MUFU / FMA counters
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
ATTN_IMPLS=${IMPLS:-51,58,59} ATTN_ROUNDS=3 timeout -s KILL 600 python tools/microbench.py attn > $O/mb_attn_diag.jsonl 2>&1; echo "mb exit $?"
for I in ${NCU_IMPLS:-51 59}; do
timeout -s KILL 300 ncu --set full --clock-control none --import-source on -k regex:attention -s 1 -c 1 \
  -o $O/attn_diag_${L:-16896}_${D:-128}_$I python tools/attn_one.py ${L:-16896} ${H:-24} ${D:-128} $I > $O/ncu_attn_diag_$I.log 2>&1; echo "ncu $I exit $?"
done
