# attention A/B (split-K/V rings) + ncu of one split-KV launch (L=16896, H=3) on A and B
cd $GRAFT_REPO_ROOT
O=gpurun_out
bash tools/gpurun_attn_ab.sh
for v in A B; do
  TSV_LIB=$PWD/build/ab/$v.so timeout -s KILL 300 ncu --set full --clock-control none --import-source on -k regex:attention -s 1 -c 1 \
    -o $O/attn_h3_$v python tools/attn_one_split.py 16896 3 128 > $O/ncu_h3_$v.log 2>&1; echo "ncu $v exit $?"
done
