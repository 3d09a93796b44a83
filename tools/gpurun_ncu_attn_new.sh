# ncu --set full of the step's attention at FLUX 2048^2 (impl 0) and the no-exp diagnostic (59)
cd $GRAFT_REPO_ROOT
O=gpurun_out
for I in ${IMPLS:-0 59}; do
timeout -s KILL 300 ncu --set full --clock-control none --import-source on -k regex:attention -s 1 -c 1 \
  -o $O/attn2_${L:-16896}_${D:-128}_$I python tools/attn_one.py ${L:-16896} ${H:-24} ${D:-128} $I > $O/ncu_attn2_$I.log 2>&1; echo "ncu $I exit $?"
done
