# ncu --set full of one attention launch.  Env: L H D IMPLS
cd $GRAFT_REPO_ROOT
O=gpurun_out
for I in ${IMPLS:-0}; do
timeout -s KILL 300 ncu --set full --clock-control none --import-source on -k regex:attention -s 1 -c 1 \
  -o $O/attn_${L:-16896}_${D:-128}_$I python tools/attn_one.py ${L:-16896} ${H:-24} ${D:-128} $I > $O/ncu_attn_$I.log 2>&1; echo "ncu $I exit $?"
done
