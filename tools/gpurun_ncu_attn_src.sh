# one attention launch under ncu --set full with source counters; the SASS-level stall sampling is
# exported on the box (CSV) and the report removed.  Env: L H D IMPL
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
T=attn_${L:-1536}_${H:-24}_${D:-128}
timeout -s KILL 300 ncu --set full --clock-control none --import-source on -k regex:attention -s 1 -c 1 \
  -o /tmp/$T python tools/attn_one.py ${L:-1536} ${H:-24} ${D:-128} ${IMPL:-0} > $O/ncu_$T.log 2>&1; echo "ncu exit $?"
ncu -i /tmp/$T.ncu-rep --page source --csv --print-source sass > $O/${T}_sass.csv 2>/dev/null; echo "src exit $?"
python tools/ncu_summary.py report /tmp/$T.ncu-rep > $O/${T}_summary.txt 2>&1
ncu -i /tmp/$T.ncu-rep --page details --csv > $O/${T}_details.csv 2>/dev/null
ls -la $O/${T}*
