# compute-sanitizer memcheck / synccheck on the tiny step (smoke) and a tiny SD3 step
cd $GRAFT_REPO_ROOT
O=gpurun_out
timeout -s KILL 600 compute-sanitizer --tool memcheck --print-limit 20 python -c "import __graft_entry__ as g; g.smoke()" > $O/sanitize_memcheck.log 2>&1; echo "memcheck $?"; tail -5 $O/sanitize_memcheck.log
timeout -s KILL 600 compute-sanitizer --tool synccheck --print-limit 20 python -c "import __graft_entry__ as g; g.smoke()" > $O/sanitize_synccheck.log 2>&1; echo "synccheck $?"; tail -5 $O/sanitize_synccheck.log
timeout -s KILL 1200 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_cases.py > $O/sanitize_cases.log 2>&1; echo "memcheck cases $?"; tail -8 $O/sanitize_cases.log
