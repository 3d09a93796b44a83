# full GPU test suite, then the whole-step A/B
cd $GRAFT_REPO_ROOT
PYARGS="-x -q" bash tools/gpurun_tests.sh
ROUNDS=${ROUNDS:-2} bash tools/gpurun_step_ab.sh
