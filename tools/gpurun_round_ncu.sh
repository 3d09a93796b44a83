# ncu evidence with the --set full reports summarised ON the box (reports are too big to copy back)
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
bash tools/gpurun_evidence.sh > $O/evidence.log 2>&1; echo "ncu exit $?"
for t in 512 2048 sd31024; do
  python tools/ncu_summary.py launches $O/launches_$t.csv > $O/launches_${t}_summary.txt 2>&1
done
python tools/ncu_summary.py report $O/prof_*.ncu-rep > $O/ncu_full_summary.txt 2>&1; echo "summary exit $?"
mkdir -p /tmp/ncu_reps && mv $O/*.ncu-rep /tmp/ncu_reps/
du -sh $O
