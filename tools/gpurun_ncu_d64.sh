# ncu --set full of the SD3 2048^2 attention (L = 16 717, H = 24, D = 64) per impl
cd $GRAFT_REPO_ROOT
O=gpurun_out
for I in ${IMPLS:-92 93 94}; do
timeout -s KILL 300 ncu --set full --clock-control none -k regex:attention -s 1 -c 1 \
  -o $O/attn_d64_$I python tools/attn_one.py 16717 24 64 $I > /dev/null 2>&1; echo "ncu $I exit $?"
done
